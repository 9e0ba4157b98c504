out=gpurun_out/$1; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1 || { tail $out/build.log; exit 1; }
for s in 64 96 128; do
TG_SB_DEFAULT=$s timeout 600 python bench.py --no-cpu-baseline --no-profile --second-precision f16x3 > $out/bench_$s.json 2> $out/bench_$s.err
python -c "import json;d=json.load(open('$out/bench_$s.json'));print($s, d['config']['superbatch'], d['value']/1e6, d['f16x3']['value']/1e6)" || tail -3 $out/bench_$s.err
done
timeout 900 python tools/next2.py --out $out/next2.json 2>&1 | tail -5
timeout 900 python tools/next3.py --out $out/next3.json 2>&1 | tail -3
