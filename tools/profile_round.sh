#!/bin/bash
# ncu evidence for the bench's step (run on the GPU box from the repo root):
#   1. launch list (gpu__time_duration per launch) of a short bench run
#   2. one `--set full` capture each of K4 (k_inject_jit) and K5 (k_classify, k_classify_slow)
#      on the bench's replica set (tools/prof_driver.py / tools/k4_time.py), raw pages as CSV
set -u
OUT=${1:-gpurun_out/prof}
mkdir -p "$OUT"
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file "$OUT/launches.csv" \
    python bench.py --steps 2 --warmup 3 --no-e2e --no-secondary --no-cpu-baseline > "$OUT/bench_under_ncu.log" 2>&1
FI_JIT_DUMP="$OUT/k4mod" ncu --set full --import-source on --clock-control none -k regex:k_inject_jit -c 1 \
    -o "$OUT/k4" python tools/k4_time.py C2 10000 1 > "$OUT/k4.log" 2>&1
ncu --set full --clock-control none -k regex:k_classify -c 2 -o "$OUT/k5" \
    python tools/prof_driver.py C2 10000 > "$OUT/k5.log" 2>&1
for r in k4 k5; do ncu -i "$OUT/$r.ncu-rep" --page raw --csv > "$OUT/${r}_raw.csv" 2>/dev/null; done
ncu -i "$OUT/k4.ncu-rep" --page source --csv --print-source sass > "$OUT/k4_source.csv" 2>/dev/null
echo done
