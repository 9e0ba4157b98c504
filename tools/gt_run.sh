out=gpurun_out/gt1; mkdir -p $out
for nk in "1032 172" "516 1032" "172 688" "172 172"; do
  set -- $nk
  for mode in 0 5; do
    echo "=== N=$1 K=$2 mode=$mode"; timeout 300 python tools/gemm_trace.py --n $1 --k $2 --precision tf32x3 --mode $mode --edges 60000 2>&1 | tail -14
  done
done > $out/trace.txt 2>&1
cat $out/trace.txt
