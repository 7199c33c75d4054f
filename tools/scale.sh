#!/bin/bash
# Strong-scaling run of bench.py on one node (for boxes with >1 GPU):
#   bash tools/scale.sh [grid] [steps] [exchange]   -> gpurun_out/scale_<grid>_<exchange>.jsonl + efficiency
# (exchange: fused | copy | nccl; every N > 1 run ends with bench's --verify of
# the chunk borders, so the first multi-GPU run also proves the cross-device
# exchange bit for bit)
# Efficiency E(N) = value(N) / (N * value(1)); every value is the
# max-over-ranks CUDA-event time of bench.py itself.
GRID=${1:-512}; STEPS=${2:-100}; EX=${3:-fused}
NGPU=$(nvidia-smi -L | wc -l)
OUT=gpurun_out/scale_${GRID}_${EX}.jsonl
mkdir -p gpurun_out; : > $OUT
for N in 1 2 4 8; do
  [ $N -gt $NGPU ] && break
  if [ $N -eq 1 ]; then
    python bench.py --grid $GRID --steps $STEPS --warmup 6 --no-e2e --no-cpu-baseline --exchange $EX >> $OUT
  else
    python -m torch.distributed.run --nnodes=1 --nproc-per-node=$N --master-addr=127.0.0.1 --master-port=$((29600+N)) \
      bench.py --gpus $N --grid $GRID --steps $STEPS --warmup 6 --no-e2e --no-cpu-baseline --exchange $EX --verify >> $OUT
  fi
done
python - $OUT <<'PY'
import json, sys
rows = [json.loads(l) for l in open(sys.argv[1]) if l.strip().startswith("{")]
v1 = rows[0]["value"]
for r in rows:
    n = r["n_gpus"]
    print("N=%d  %.4g node-updates/s  %.3f ms/step  efficiency %.3f  halo wait %s  verify %s" % (
        n, r["value"], r["ms_per_step"], r["value"] / (n * v1), r["halo"]["measured_wait_ms_per_launch"],
        r.get("verify", {}).get("ok")))
PY
