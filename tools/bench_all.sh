# One bench line per BASELINE.json workload (1 GPU): configs[0..4]. Usage: bash tools/bench_all.sh outdir
out=${1:-gpurun_out/bench_all}; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for c in config1 wiki mooc lastfm large; do
  extra="--no-cpu-baseline"
  [ "$c" = "config1" ] && extra=""
  timeout 1200 python bench.py --config $c --steps 3 --warmup 3 $extra > $out/bench_$c.json 2> $out/bench_$c.err
  python -c "import json;d=json.load(open('$out/bench_$c.json'));print('$c', round(d['value']/1e6,3), 'M edges/s', round(d['ms_per_step'],1), 'ms', 'bf16', round(d['bf16']['value']/1e6,3), 'S', d['config']['superbatch'], 'hit', d['stats']['hit_rate_mean_of_batches'], 'dedup', d['stats']['dedup_ratio'], 'roof', d['roofline']['kernel'], round(d['roofline']['frac'],3))" || tail -3 $out/bench_$c.err
done
