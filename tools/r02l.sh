out=gpurun_out/$1; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1 || { tail $out/build.log; exit 1; }
for pp in 1 0; do
TG_PHI_PRE=$pp timeout 600 python bench.py --no-cpu-baseline --no-profile --second-precision f16x3 > $out/bench_pp$pp.json 2> $out/bench_pp$pp.err
python -c "import json;d=json.load(open('$out/bench_pp$pp.json'));print('phi_pre', $pp, d['value']/1e6, d['f16x3']['value']/1e6)" || tail -3 $out/bench_pp$pp.err
done
