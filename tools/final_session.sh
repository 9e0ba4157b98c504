#!/bin/bash
# Round-end evidence: build, all GPU tests, smoke, bench line (with cpu_baseline), ncu launch
# list of the bench, ncu --set full of the attention kernel, NEXT-1 / NEXT-4 sweeps.
tag=${1:-final}; out=gpurun_out/$tag; mkdir -p $out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $out/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1 || { tail -20 $out/build.log; exit 1; }
timeout 1800 python -m pytest tests -q -m gpu > $out/tests.log 2>&1; echo "tests rc=$?"; tail -3 $out/tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $out/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $out/smoke.log
timeout 900 python bench.py > $out/bench.json 2> $out/bench.err; echo "bench rc=$?"; python -c "import json;d=json.load(open('$out/bench.json'));print(d['value'],d['ms_per_step'],d['e2e']['value'],d['roofline']['frac'],d['cpu_baseline']['value'])"
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > $out/bench_reference.json 2> $out/bench_reference.err; echo "ref rc=$?"; tail -c 300 $out/bench_reference.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 5000 --csv --log-file $out/launches.csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-profile > $out/launches_bench.log 2>&1; echo "launches rc=$?"
python tools/launch_summary.py $out/launches.csv --json $out/launches_summary.json > /dev/null 2>&1; python tools/sb_launches.py $out/launches.csv > $out/superbatch_launches.txt 2>&1; tail -18 $out/superbatch_launches.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_attn_g -s 200 -c 1 -o $out/attn python tools/profile_run.py > $out/full_attn.log 2>&1; echo "full attn rc=$?"
python tools/ncu_summary.py $out/attn.ncu-rep > $out/attn.summary.txt 2>&1; python tools/ncu_lines.py $out/attn.ncu-rep --top 40 > $out/attn.lines.txt 2>&1; python tools/ncu_stalls.py $out/attn.ncu-rep > $out/attn.stalls.txt 2>&1; head -c 700 $out/attn.summary.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gemm_tc -s 361 -c 1 -o $out/gemm python tools/profile_run.py > $out/full_gemm.log 2>&1; echo "full gemm rc=$?"
python tools/ncu_summary.py $out/gemm.ncu-rep > $out/gemm.summary.txt 2>&1; head -c 400 $out/gemm.summary.txt
timeout 1200 python tools/sweep.py --out $out/sweep_L2k20.json > $out/sweep_L2.log 2>&1; echo "sweep L2 rc=$?"
timeout 1200 python tools/sweep.py --model 3,8 --passes 2 --out $out/sweep_L3k8.json > $out/sweep_L3.log 2>&1; echo "sweep L3 rc=$?"
