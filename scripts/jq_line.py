"""Print the key numbers of a bench.py JSON line read from stdin."""
import json
import sys

for line in sys.stdin:
    if line.startswith("{"):
        d = json.loads(line)
        r = d.get("roofline") or {}
        s = d.get("setup") or {}
        print("%s value %.4g %s kern %s ms frac %s variant %s smem %s" % (
            d["config"].get("workload", "")[:24], d["value"], d["unit"], r.get("kernel_ms_avg"), r.get("frac"),
            s.get("eval_variant"), s.get("smem_bytes")))
    elif "rror" in line:
        print(line.strip()[:300])
