set -x
python tools/exp_options.py --sweeps 5 --set "filter32=0" --set "filter32=1" --set "chunk_tokens=8192" 2>&1 | grep -v "^#"
for v in ring4 ring2 match minb2; do LDA_LIBRARY=$PWD/variants/$v.so python tools/exp_options.py --sweeps 5 --set "filter32=0" 2>&1 | grep -v "^#" | sed "s/^/$v /"; done
