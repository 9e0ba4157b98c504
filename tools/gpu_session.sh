#!/bin/bash
# One GPU session: build, gpu tests, smoke, bench, ncu launch list and full captures.
# usage: bash tools/gpu_session.sh [tag] [what...]   (what: tests smoke bench launches full)
tag=${1:-r01}; shift
what=${@:-tests smoke bench launches full}
out=gpurun_out/$tag; mkdir -p $out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $out/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1 || { tail -20 $out/build.log; exit 1; }
for w in $what; do case $w in
 tests) timeout 900 python -m pytest tests -x -q -m gpu > $out/tests.log 2>&1; echo "tests rc=$?"; tail -3 $out/tests.log;;
 smoke) timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $out/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 $out/smoke.log;;
 bench) timeout 900 python bench.py > $out/bench.json 2> $out/bench.err; echo "bench rc=$?"; tail -c 3000 $out/bench.json;;
 launches) timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 100000 --csv --log-file $out/launches.csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-profile > $out/launches_bench.log 2>&1; echo "launches rc=$?"; python tools/launch_summary.py $out/launches.csv --json $out/launches_summary.json > /dev/null 2>&1; head -c 2500 $out/launches_summary.json;;
 benchq) timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > $out/benchq.json 2> $out/benchq.err; echo "benchq rc=$?"; python -c "import json;d=json.load(open('$out/benchq.json'));print(d['value'],d['ms_per_step'],d['roofline']['avg_launch_us'],d['stages_ms'])";;
 fullattn) timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_attn -s 200 -c 1 -o $out/attn python tools/profile_run.py > $out/full_attn.log 2>&1; echo "full attn rc=$?"
       python tools/ncu_summary.py $out/attn.ncu-rep > $out/attn.summary.txt 2>&1; cat $out/attn.summary.txt; python tools/ncu_lines.py $out/attn.ncu-rep --top 40 > $out/attn.lines.txt 2>&1; python tools/ncu_stalls.py $out/attn.ncu-rep > $out/attn.stalls.txt 2>&1; cat $out/attn.stalls.txt;;
 full) timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_attn -s 200 -c 2 -o $out/attn python tools/profile_run.py > $out/full_attn.log 2>&1; echo "full attn rc=$?"
       timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gemm_tc -s 400 -c 4 -o $out/gemm python tools/profile_run.py > $out/full_gemm.log 2>&1; echo "full gemm rc=$?"
       for r in attn gemm; do python tools/ncu_summary.py $out/$r.ncu-rep > $out/$r.summary.txt 2>&1; cat $out/$r.summary.txt; done;;
esac; done
