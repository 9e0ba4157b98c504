# env-knob A/B of the GEMM plan on the tf32x3 bench (e.g. TG_GEMM_STG / TG_GEMM_SB): "name:VAR=v,VAR=v" ...
out=gpurun_out/$1; shift; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1 || { tail $out/build.log; exit 1; }
for spec in default "$@"; do
  name=${spec%%:*}; envs=""; [ "$spec" != default ] && envs=$(echo ${spec#*:} | tr ',' ' ')
  for prec in tf32x3 f16x3; do
    env $envs timeout 600 python bench.py --steps 5 --warmup 3 --precision $prec --second-precision none --no-cpu-baseline > $out/b_${name}_$prec.json 2> $out/b_${name}.err
    python - $out/b_${name}_$prec.json "$name $prec" <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l); rk=d['roofline_kernels']
        print(f"{sys.argv[2]:22s} {d['value']/1e6:.3f} M  ms {d['ms_per_step']:.2f}  " + " ".join(f"{k.split()[-1]}={v['avg_launch_us']:.1f}" for k,v in rk.items()))
PY
  done
done
