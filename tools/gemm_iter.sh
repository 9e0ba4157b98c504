# GEMM iteration: build, GEMM + parity subset, tf32x3/f16x3 bench line, clock64 traces of the 4 GEMM shapes
tag=$1; out=gpurun_out/$tag; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1 || { tail $out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q -k "gemm or ln_fused or embed or stream_scores or fullsize_reddit or superbatch_invariance or f16x3" > $out/tests.log 2>&1; tail -3 $out/tests.log
timeout 600 python bench.py --steps 5 --warmup 3 --second-precision bf16,f16x3 --no-cpu-baseline > $out/bench.json 2> $out/bench.err; tail -c 400 $out/bench.err
python - $out/bench.json <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l); print('value', d['value'], 'ms', d['ms_per_step'], 'e2e', d['e2e']['value'], 'bf16', d.get('bf16',{}).get('value'), 'f16x3', d.get('f16x3',{}).get('value'))
        for k,v in d['roofline_kernels'].items(): print(' ', k, round(v['achieved'],1), round(v['frac'],3), round(v['share_of_step'],3), round(v['avg_launch_us'],1))
PY
for nk in "1032 172" "516 1032" "172 688" "172 172"; do
  set -- $nk
  for mode in 0 5; do
    echo "=== N=$1 K=$2 mode=$mode"; timeout 300 python tools/gemm_trace.py --n $1 --k $2 --precision tf32x3 --mode $mode --edges 60000 2>&1 | grep -v "^unit [67]" | tail -12
  done
done > $out/trace.txt 2>&1
grep -A3 "===\|epi_\|mma_done" $out/trace.txt | head -80
