#!/bin/bash
# NVLink cross-check of the library's link-byte counters (bytes_link_remote) on a multi-GPU box.
# Reads every GPU's NVLink data counters (nvidia-smi nvlink -gt d: KiB transmitted / received per
# link) before and after one multi-process run, and prints the per-GPU deltas next to the bench
# line's per-loop link bytes. ncu cannot profile a multi-rank command (it replays kernels), so the
# driver-level counters are the evidence here.
# Usage: scripts/nvlink_counters.sh N [bench args...]      e.g. scripts/nvlink_counters.sh 8 --steps 50
set -e
N=${1:-2}; shift || true
OUT=${OUT:-gpurun_out/nvlink}
mkdir -p $OUT
nvidia-smi nvlink -gt d > $OUT/before.txt 2>&1 || { echo "nvidia-smi nvlink unavailable"; exit 0; }
python bench.py --gpus $N --no-e2e --no-cpu-baseline "$@" > $OUT/bench.jsonl
nvidia-smi nvlink -gt d > $OUT/after.txt 2>&1
python - "$OUT" <<'PY'
import json, re, sys
out = sys.argv[1]
def parse(path):
    gpu, tot = None, {}
    for line in open(path):
        m = re.match(r"GPU (\d+):", line)
        if m:
            gpu = int(m.group(1)); tot.setdefault(gpu, [0, 0]); continue
        m = re.search(r"Link \d+: Data Tx: (\d+) KiB", line)
        if m and gpu is not None: tot[gpu][0] += int(m.group(1))
        m = re.search(r"Link \d+: Data Rx: (\d+) KiB", line)
        if m and gpu is not None: tot[gpu][1] += int(m.group(1))
    return tot
b, a = parse(f"{out}/before.txt"), parse(f"{out}/after.txt")
line = json.loads(open(f"{out}/bench.jsonl").read().strip().splitlines()[-1])
print(json.dumps({"nvlink_tx_bytes": {g: (a[g][0] - b[g][0]) * 1024 for g in a},
                  "nvlink_rx_bytes": {g: (a[g][1] - b[g][1]) * 1024 for g in a},
                  "bench_steps": line.get("steps"), "bench_warmup": line.get("warmup"),
                  "library_link_bytes_per_loop": line.get("link_bytes_per_loop"),
                  "library_link_remote_bytes_per_loop": line.get("link_remote_bytes_per_loop")}))
PY
