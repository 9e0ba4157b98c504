for nk in "516 1032" "172 688" "1032 172"; do set -- $nk; echo "== N=$1 K=$2"; python tools/gemm_trace.py --n $1 --k $2 --precision tf32x3 --edges 60000 --mode 3 2>&1 | grep -E "mma_full|prod_"; done
