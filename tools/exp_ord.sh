cd "$(dirname "$0")/.."
for m in 0 1 2 3; do export HDB_ORD_MASK=$m; echo "ORD_MASK=$m"; SEL=kernel_variant WLS="C2-eps0.45 C2-eps1.40 C5-eps0.5" bash tools/exp_quick.sh | grep ms; done
