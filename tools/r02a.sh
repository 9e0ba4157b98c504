out=gpurun_out/r02a; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
for p in tf32x3 bf16; do
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --precision $p > $out/bench_$p.json 2> $out/bench_$p.err
python -c "import json;d=json.load(open('$out/bench_$p.json'));print('$p', round(d['value']/1e6,3), 'M edges/s', round(d['ms_per_step'],2), 'ms e2e', round(d['e2e']['value']/1e6,3), d['stages_ms'])" || tail -5 $out/bench_$p.err
done
