#!/bin/bash
# ncu evidence for one round (run on the GPU box from the repo root):
#   bash tools/ncu_capture.sh <tag>
# 1. launch list of one 32-layer bench step (serialised, cold-cache per-launch times)
# 2. `--set full` captures of the dominant kernels on a 2-layer model of the same shapes
set -u
TAG=${1:-r1d}
OUT=gpurun_out
mkdir -p $OUT
if [ "${SKIP_LAUNCHES:-0}" != 1 ]; then
ncu --metrics gpu__time_duration.sum --clock-control none --nvtx --nvtx-include "step/" --csv \
    --log-file $OUT/launches_$TAG.csv python tools/profile_step.py --steps 1 > $OUT/ncu_launch_$TAG.log 2>&1
fi
cap() {  # name, kernel regex, skip
  QOS_OVERLAP_ATTN=0 ncu --set full --clock-control none --import-source on --nvtx --nvtx-include "step/" \
      --kernel-name-base demangled -k "regex:$2" -s "$3" -c 1 -o $OUT/prof_${1}_$TAG \
      python tools/profile_step.py --steps 1 --layers 2 > $OUT/ncu_${1}_$TAG.log 2>&1
}
# GEMM launches per layer at T = 2176: QKV(+RoPE), O and down on the CTA-pair kernel
# (gemm2_tcgen05_kernel: layer 1 QKV = 3, O = 4; layer 0 down = 2, whose epilogue carries the folded
# norm), gate/up on the single-CTA tile kernel
# (gemm_tcgen05_kernel: layer 1 = launch 1)
if [ "${ONLY_ATTN:-0}" != 1 ]; then
cap gemm_qkv_rope 'gemm2_tcgen05_kernel' 3
cap gemm_o 'gemm2_tcgen05_kernel' 4
cap gemm_down 'gemm2_tcgen05_kernel' 2
cap gemm_gateup 'gemm_tcgen05_kernel' 1
fi
if [ "${ONLY_GEMM:-0}" != 1 ]; then
cap decode_attn 'decode_attn_kernel' 1
cap prefill_attn 'prefill_attn_(tc|persist)_kernel' 1
fi
ls -la $OUT
