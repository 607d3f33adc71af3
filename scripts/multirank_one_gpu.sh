#!/bin/bash
# The N > 1 bench path (shards, fused P2P Sync over CUDA IPC, max-over-ranks timing, JSON line) run
# as 2 ranks sharing ONE GPU (LOWDIFF_BENCH_DEVICE=0): a liveness/contract check only — the two
# contexts time-slice the device, so the numbers say nothing about NVLink scaling.
# Usage (GPU box): bash scripts/multirank_one_gpu.sh [config] [extra bench args...]
C=${1:-1}; shift
OUT=gpurun_out; mkdir -p $OUT
LOWDIFF_P2P_TIMEOUT_MS=${LOWDIFF_P2P_TIMEOUT_MS:-20000} LOWDIFF_BENCH_DEVICE=0 timeout 900 \
  python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 \
  bench.py --gpus 2 --config $C --steps 2 --warmup 3 "$@" > $OUT/multirank_C$C.json 2> $OUT/multirank_C$C.err
echo "multirank C$C rc=$?"; tail -c 1500 $OUT/multirank_C$C.json; tail -3 $OUT/multirank_C$C.err
