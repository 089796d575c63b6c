#!/bin/bash
# bench each library variant in variants/ (sampler 0) + the default build
for f in variants/*.so; do
  echo "== $f"
  LDA_LIBRARY=$PWD/$f python bench.py --steps 5 --warmup 3 --no-cpu-baseline 2>&1 | python tools/brief.py
done
