"""B200-native HYBRID-DBSCAN hot path (Gowanlock et al., IPDPSW 2017).

The product is ``libhdb.so`` (CUDA sm_100a kernels + C++ host orchestration)
behind the C-ABI in ``include/hdb.h``; :mod:`.hdb` is its ctypes binding.
"""
import os

PKG_DIR = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(PKG_DIR, "libhdb.so")


def build(verbose: bool = False) -> str:
    """Compile libhdb.so in-tree for sm_100a (make -C csrc)."""
    import subprocess
    cmd = ["make", "-C", os.path.join(PKG_DIR, "csrc"), f"-j{os.cpu_count() or 4}"]
    r = subprocess.run(cmd, capture_output=not verbose, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"libhdb build failed:\n{r.stdout}\n{r.stderr}")
    return LIB_PATH
