python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1500 python -m pytest tests -q -m gpu -x 2>&1 | tail -3
bash tools/bench_all.sh gpurun_out/r02w
timeout 600 python tools/next3.py --out gpurun_out/r02w/next3.json 2>&1 | tail -2
