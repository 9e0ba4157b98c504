tag=$1; out=gpurun_out/$tag; mkdir -p $out
bash tools/r02_full.sh $tag
bash tools/r02_profile.sh $tag tf32x3
