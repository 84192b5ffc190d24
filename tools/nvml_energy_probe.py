"""How often does NVML's total-energy counter advance on this GPU?  (The
bench's overlap probes read it around each run; sub-second runs are only as
good as its update interval.)  Prints one JSON line."""
import json
import time

import pynvml

pynvml.nvmlInit()
h = pynvml.nvmlDeviceGetHandleByIndex(0)
t_end = time.time() + 3.0
last, changes, vals = None, [], []
while time.time() < t_end:
    e = pynvml.nvmlDeviceGetTotalEnergyConsumption(h)
    t = time.perf_counter()
    if last is not None and e != last:
        changes.append(t)
    last = e
    vals.append(e)
gaps = [b - a for a, b in zip(changes, changes[1:])]
print(json.dumps({"reads": len(vals), "changes": len(changes),
                  "median_update_interval_ms": 1e3 * sorted(gaps)[len(gaps) // 2] if gaps else None,
                  "max_update_interval_ms": 1e3 * max(gaps) if gaps else None}))
