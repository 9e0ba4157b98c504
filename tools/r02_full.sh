# GPU session: tests, smoke, bench (usage: bash tools/r02_full.sh tag)
tag=$1; out=gpurun_out/$tag; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1 || { tail -20 $out/build.log; exit 1; }
timeout 1500 python -m pytest tests -q -m gpu -rA --durations=15 > $out/tests.log 2>&1; echo "tests rc=$?"; grep -E "passed|failed" $out/tests.log | tail -3
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $out/smoke.log 2>&1; echo "smoke rc=$?"; tail -3 $out/smoke.log
timeout 900 python bench.py > $out/bench.json 2> $out/bench.err; echo "bench rc=$?"
python -c "import json;d=json.load(open('$out/bench.json'));print(d['dtype'], d['value']/1e6, d['ms_per_step'], 'e2e', d['e2e']['value']/1e6, 'bf16', d['bf16']['value']/1e6, d['roofline']['kernel'], d['roofline']['frac'], d['stats']['dedup_ratio'], d['stats']['hit_rate_mean_of_batches'])" || tail -5 $out/bench.err
