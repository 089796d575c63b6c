# A/B of compile-time variants (variants/liblda_<name>.so) on the bench workload
# usage: bash tools/gpu_variants.sh <tag> <config> name1 name2 ...
tag=$1; cfg=$2; shift 2
mkdir -p gpurun_out
for v in "$@"; do
  for rep in 1 2; do
    LDA_LIBRARY=variants/liblda_$v.so timeout 600 python tools/exp_options.py --config $cfg --sweeps 10 --warmup 25 \
      2>&1 | grep -v "^#" | sed "s/^/$v /" >> gpurun_out/${tag}_variants.log
  done
done
cat gpurun_out/${tag}_variants.log
