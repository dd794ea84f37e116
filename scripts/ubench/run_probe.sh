#!/bin/bash
# FP32 pipe / isolated K1 loop micro-benchmarks (build on the box, run, log to gpurun_out/)
cd "$(dirname "$0")"
mkdir -p ../../gpurun_out/probe
for b in ffma2 loop2d; do
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr -o /tmp/$b $b.cu && timeout 120 /tmp/$b > ../../gpurun_out/probe/$b.txt 2>&1
  echo "$b rc=$?"; cat ../../gpurun_out/probe/$b.txt
done
