# GEMM clock64 traces (debug build libtg_trace.so) of the layer GEMM shapes, tf32x3
out=gpurun_out/$1; mkdir -p $out
for nk in ${SHAPES:-"516 1032" "1032 172" "172 688" "172 172"}; do
  set -- $nk
  for mode in ${MODES:-0 3 5}; do
    echo "=== N=$1 K=$2 mode=$mode"; timeout 300 python tools/gemm_trace.py --n $1 --k $2 --precision tf32x3 --mode $mode --edges 60000 2>&1 | tail -14
  done
done > $out/trace.txt 2>&1
cat $out/trace.txt
