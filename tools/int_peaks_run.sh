#!/bin/bash
# Integer-pipe peaks with the SM clock recorded during the run (run under gpurun).
# writes gpurun_out/int_peaks.json (copy to profiles/int_peaks.json when accepted)
mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/int_peaks tools/int_peaks.cu || exit 1
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active \
  --format=csv,noheader,nounits -lms 50 > /tmp/int_peaks_clk.csv 2>/dev/null &
SMI=$!
sleep 0.5
/tmp/int_peaks > /tmp/int_peaks.json 2> gpurun_out/int_peaks.log
kill $SMI 2>/dev/null; wait $SMI 2>/dev/null
python - <<'PY'
import json
d = json.load(open("/tmp/int_peaks.json"))
rows = [l.split(",") for l in open("/tmp/int_peaks_clk.csv") if l.strip()]
load = sorted(float(r[0]) for r in rows if float(r[2]) > 300.0) or sorted(float(r[0]) for r in rows)
d["clocks"] = {"sm_mhz_median_under_load": load[len(load) // 2] if load else None,
               "sm_max_mhz": float(rows[0][1]) if rows else None, "samples": len(rows),
               "reasons_seen": sorted({r[3].strip() for r in rows})}
json.dump(d, open("gpurun_out/int_peaks.json", "w"))
print(json.dumps(d))
PY
