# compute-sanitizer racecheck / synccheck / memcheck of one small stream pass (config1 prefix)
out=gpurun_out/$1; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for tool in memcheck racecheck synccheck; do
  for p in tf32x3 bf16; do
    timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/profile_run.py --config config1 --precision $p --edges 4000 > $out/${tool}_$p.log 2>&1
    echo "$tool $p rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' $out/${tool}_$p.log | tail -2 | tr '\n' ' ')"
  done
done
