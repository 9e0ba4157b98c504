out=gpurun_out/$1; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x 2>&1 | tail -3
for p in tf32x3 f16x3; do
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/launches_$p.csv -s 2000 -c 300 python tools/profile_run.py --precision $p > /dev/null 2>&1
python tools/sb_launches.py $out/launches_$p.csv > $out/sb_$p.txt 2>&1; head -28 $out/sb_$p.txt | grep -E "gemm|total"
done
python bench.py --no-cpu-baseline --precision tf32x3 --second-precision f16x3 > $out/bench.json 2> $out/bench.err; python -c "import json;d=json.load(open('$out/bench.json'));print(d['value']/1e6, d['stages_ms']); print(d['f16x3']['value']/1e6, d['f16x3']['stages_ms'])" || tail $out/bench.err
