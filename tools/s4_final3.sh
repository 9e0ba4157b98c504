# final session part 3: ncu launch list of a whole pass + ncu --set full of ~one superbatch (kernel
# table: DRAM GB/s per kernel, tensor-pipe activity per GEMM), then compute-sanitizer on config1
tag=$1; prec=${2:-tf32x3}; out=gpurun_out/$tag; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1 || { tail $out/build.log; exit 1; }
timeout 900 ncu --metrics gpu__time_duration.sum,launch__grid_size --clock-control none --csv --log-file $out/launches_$prec.csv python tools/profile_run.py --precision $prec > /dev/null 2>&1; echo "launches rc=$?"
python tools/launch_summary.py $out/launches_$prec.csv --json $out/launches_summary_$prec.json > /dev/null 2>&1
python tools/sb_launches.py $out/launches_$prec.csv > $out/sb_$prec.txt 2>&1; tail -32 $out/sb_$prec.txt
timeout 1500 ncu --set full --clock-control none --import-source on -s 400 -c 36 -o $out/sb_full_$prec python tools/profile_run.py --precision $prec > $out/full_$prec.log 2>&1; echo "full rc=$?"
python tools/kernel_table.py $out/sb_full_$prec.ncu-rep --out $out/kernels_$prec --tag $prec 2>&1 | tail -40
python tools/ncu_summary.py $out/sb_full_$prec.ncu-rep --json $out/sb_full_$prec.summary.json > /dev/null
ncu -i $out/sb_full_$prec.ncu-rep --page source --csv --print-source sass -k regex:k_attn_g > $out/attn_src.csv 2>/dev/null; gzip -f $out/attn_src.csv
gzip -f $out/launches_$prec.csv; rm -f $out/sb_full_$prec.ncu-rep
[ -n "$SANITIZE" ] && bash tools/sanitize.sh $tag
