#!/bin/bash
# NVLink / HBM evidence for the multi-GPU CPU-Free runs on an 8-GPU node (nsys is not in this
# image; run where it is installed).  ncu cannot profile the cross-GPU persistent kernels (it
# serialises kernels, so the GPUs' flag waits would never be satisfied — the watchdog fires),
# so the per-GPU DRAM bandwidth and NVLink throughput are sampled with nsys GPU metrics, which
# do not serialise:
#
#   scripts/nsys_nvlink.sh [N] [config]
#
# then read the "NVLink RX/TX" and "DRAM Read/Write Bandwidth" rows of the report per GPU; the
# halo bytes per iteration the bench line states (`halo_traffic`) times iterations per second is
# the expected NVLink traffic.
N=${1:-8}
CFG=${2:-c2}
OUT=${OUT:-gpurun_out/nsys_${CFG}_n${N}}
nsys profile --gpu-metrics-devices=all --gpu-metrics-set=gb200 --gpu-metrics-frequency=20000 \
     --trace=cuda,nvtx --output "$OUT" --force-overwrite true \
     python bench.py --gpus "$N" --config "$CFG" --steps 3 --warmup 3 --no-extras
nsys stats --report gpu_metrics_summary "$OUT.nsys-rep" 2>/dev/null || nsys stats "$OUT.nsys-rep"
