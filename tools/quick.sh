#!/bin/bash
# Quick GPU iteration: build, parity tests, bench line, one superbatch's launch list (ncu).
# usage: bash tools/quick.sh tag [notest] [nolaunch]
tag=$1; shift
out=gpurun_out/$tag; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1 || { tail -20 $out/build.log; exit 1; }
if [[ " $* " != *" notest "* ]]; then
  timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu > $out/tests.log 2>&1; echo "tests rc=$?"; tail -1 $out/tests.log
fi
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > $out/bench.json 2> $out/bench.err
python -c "import json;d=json.load(open('$out/bench.json'));print('bench', round(d['value']/1e6,3), 'M edges/s', round(d['ms_per_step'],2), 'ms e2e', round(d['e2e']['value']/1e6,3), d['stages_ms'])" || tail -5 $out/bench.err
if [[ " $* " != *" nolaunch "* ]]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/launches.csv -s 2000 -c 300 python tools/profile_run.py > /dev/null 2>&1
  python tools/sb_launches.py $out/launches.csv
fi
