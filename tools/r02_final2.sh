tag=$1; out=gpurun_out/$tag; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
bash tools/bench_all.sh $out
timeout 900 python tools/next2.py --out $out/next2.json 2>&1 | tail -4
timeout 900 python tools/next3.py --out $out/next3.json 2>&1 | tail -2
timeout 1500 python tools/sweep.py --out $out/sweep_L2k20.json > $out/sweep.log 2>&1; echo "sweep rc=$?"
timeout 1500 python tools/sweep.py --model 3,8 --out $out/sweep_L3k8.json > $out/sweep38.log 2>&1; echo "sweep38 rc=$?"
python tools/parity_errors.py --prec 0 1 4 2 3 --out $out/parity_errors.json 2>&1 | tail -5
