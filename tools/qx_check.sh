#!/bin/bash
# Bounds-checked k_qlanes (ab/libhdb_qxcheck.so, built with -DHDB_QX_CHECK) over the parity
# tests that reach it: the query-lane tests and the full-size C5 table.  Usage (gpurun): bash tools/qx_check.sh TAG
cd "$(dirname "$0")/.."
T=${1:-qx}
HDB_LIB=ab/libhdb_qxcheck.so timeout 1500 python -m pytest tests -m gpu -q -k "query_lane or C5" -p no:cacheprovider \
    > gpurun_out/${T}_qx_check.txt 2>&1
echo "qx_check rc=$? $(tail -1 gpurun_out/${T}_qx_check.txt)"; grep -c "bound check failed" gpurun_out/${T}_qx_check.txt
