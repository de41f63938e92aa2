#!/bin/bash
# Build the microbenchmarks on demand into tools/micro/build/ (git-ignored).
set -e
cd "$(dirname "$0")"
mkdir -p build
for f in latency random_sectors zerocopy hostlink split; do
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/$f $f.cu -lpthread -lcuda
done
