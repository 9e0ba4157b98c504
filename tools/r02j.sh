out=gpurun_out/$1; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1 || { tail $out/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x 2>&1 | tail -4
for s in 28 48 64; do
TG_SB_DEFAULT=$s timeout 600 python bench.py --no-cpu-baseline --no-profile --second-precision f16x3 > $out/bench_$s.json 2> $out/bench_$s.err
python -c "import json;d=json.load(open('$out/bench_$s.json'));print($s, d['config']['superbatch'], d['value']/1e6, d['f16x3']['value']/1e6)" || tail -3 $out/bench_$s.err
done
