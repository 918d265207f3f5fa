#!/bin/bash
# Round profiling on the GPU box (run under gpurun).  Produces, in gpurun_out/:
#   launches_<cfg>.csv   -- every launch with gpu__time_duration (cold, serialised)
#   ncu_<cfg>_summary.json -- per-kernel dram bytes / duration / issue / occupancy
#                             (one `ncu --set full` pass over one bench step)
# Usage: scripts/profile_round.sh <cfg> [bench args]
set -u
cfg=$1; shift
mkdir -p gpurun_out /tmp/prof
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_${cfg}.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu "$@" \
    > gpurun_out/launches_${cfg}.log 2>&1
# full set on the hot-path kernels of one measured step (skip the warm-up step)
timeout 1500 ncu --set full --clock-control none --import-source on \
    -k regex:'k_getrf|k_getrs|k_extract|k_plan|k_scan' -o /tmp/prof/full_${cfg} -f \
    python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu "$@" > gpurun_out/full_${cfg}.log 2>&1
ncu -i /tmp/prof/full_${cfg}.ncu-rep --page raw --csv > /tmp/prof/full_${cfg}_raw.csv 2>/dev/null
python3 - "$cfg" <<'PY'
import csv, json, sys
cfg = sys.argv[1]
rows = list(csv.reader(open(f"/tmp/prof/full_{cfg}_raw.csv")))
hdr, units, data = rows[0], rows[1], rows[2:]
want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "smsp__thread_inst_executed_per_inst_executed.ratio",
        "smsp__inst_executed.sum"]
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6, "msecond": 1e-3}
out = []
for r in data:
    d = dict(zip(hdr, r)); u = dict(zip(hdr, units))
    rec = {"kernel": d.get("Kernel Name", "")[:120]}
    for w in want:
        if w in d:
            try:
                v = float(d[w].replace(",", ""))
            except ValueError:
                continue
            rec[w] = v * scale.get(u.get(w, ""), 1)
    out.append(rec)
json.dump(out, open(f"gpurun_out/ncu_{cfg}_summary.json", "w"), indent=1)
PY
