# iteration: build, parity subset, tf32x3 (+bf16) bench line, optional ncu of one k_attn_g launch
# usage: bash tools/s3_iter.sh <tag> [ncu]
tag=$1; out=gpurun_out/$tag; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1 || { tail $out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q -k "${TESTK:-embed or stream_scores or fullsize_reddit or superbatch_invariance or opts_invariance or score_pairs or counters}" > $out/tests.log 2>&1; tail -3 $out/tests.log
timeout 600 python bench.py --steps 5 --warmup 3 --second-precision bf16 --no-cpu-baseline > $out/bench.json 2> $out/bench.err; tail -c 600 $out/bench.err
python - $out/bench.json <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l); print('value', d['value'], 'ms', d['ms_per_step'], 'e2e', d['e2e']['value'], 'bf16', d.get('bf16',{}).get('value'))
        for k,v in d['roofline_kernels'].items(): print(' ', k, round(v['achieved'],1), round(v['frac'],3), round(v['share_of_step'],3), round(v['avg_launch_us'],1))
        print(' stages', d['stages_ms'])
PY
if [ "$2" = ncu ]; then
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_attn_g -s 6 -c 2 -o $out/attn python tools/profile_run.py --precision tf32x3 > $out/ncu.log 2>&1; echo "ncu rc=$?"
python tools/ncu_summary.py $out/attn.ncu-rep --json $out/attn.summary.json > $out/attn.summary.txt 2>&1; head -60 $out/attn.summary.txt
python tools/ncu_stalls.py $out/attn.ncu-rep > $out/attn.stalls.txt 2>&1; cat $out/attn.stalls.txt | head -30
ncu -i $out/attn.ncu-rep --page source --csv --print-source sass > $out/attn_src.csv 2>/dev/null; gzip -f $out/attn_src.csv
fi
