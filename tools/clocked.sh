#!/bin/bash
# Run a command with nvidia-smi clock / throttle sampling beside it (every 100 ms):
#   tools/clocked.sh NAME CMD...   -> gpurun_out/clocks_NAME.csv + a one-line summary appended to it
name=$1; shift
mkdir -p gpurun_out
out=gpurun_out/clocks_$name.csv
nvidia-smi --query-gpu=timestamp,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap \
  --format=csv,noheader,nounits -lms 100 > $out 2>/dev/null &
smi=$!
"$@"
rc=$?
kill $smi 2>/dev/null; wait $smi 2>/dev/null
python - "$out" <<'PY'
import sys
rows = [l.split(",") for l in open(sys.argv[1]) if l.count(",") >= 7]
sm = sorted(float(r[1]) for r in rows if r[1].strip().replace(".", "").isdigit())
names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
act = sorted({names[i] for r in rows for i in range(4) if r[4 + i].strip() == "Active"})
med = sm[len(sm) // 2] if sm else None
open(sys.argv[1], "a").write(f"# summary: samples {len(rows)} sm_mhz_median {med} sm_mhz_min {sm[0] if sm else None} reasons {act}\n")
print(f"clocks: samples {len(rows)} median SM {med} MHz, min {sm[0] if sm else None}, reasons {act}")
PY
exit $rc
