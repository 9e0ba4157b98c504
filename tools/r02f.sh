out=gpurun_out/r02f; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > /dev/null
for p in f16x3 tf32x3; do
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/launches_$p.csv -s 2000 -c 300 python tools/profile_run.py --precision $p > /dev/null 2>&1
python tools/sb_launches.py $out/launches_$p.csv > $out/sb_$p.txt 2>&1; head -30 $out/sb_$p.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gemm_tc -s 400 -c 4 -o $out/gemm_$p python tools/profile_run.py --precision $p > $out/full_gemm_$p.log 2>&1
python tools/ncu_summary.py $out/gemm_$p.ncu-rep > $out/gemm_$p.summary.txt 2>&1; cat $out/gemm_$p.summary.txt
done
