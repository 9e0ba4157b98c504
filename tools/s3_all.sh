# quick bench lines (tf32x3 + bf16) per workload with the default superbatch; usage: bash tools/s3_all.sh tag [configs]
out=gpurun_out/$1; shift; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for c in ${@:-reddit config1 wiki mooc lastfm large}; do
  timeout 1200 python bench.py --config $c --steps 3 --warmup 3 --no-cpu-baseline --second-precision ${PREC2:-bf16} > $out/bench_$c.json 2> $out/bench_$c.err
  python -c "import json;d=json.load(open('$out/bench_$c.json'));print('$c', round(d['value']/1e6,3), 'M edges/s', round(d['ms_per_step'],1), 'ms', 'bf16', round(d.get('bf16',{}).get('value',0)/1e6,3), 'S', d['config']['superbatch'], 'roof', d['roofline']['kernel'], round(d['roofline']['frac'],3))" || tail -3 $out/bench_$c.err
done
