"""Record the DRAM traffic of one eval launch from an ncu --set full report:
python scripts/ncu_traffic_update.py REPORT CFG K OUT_JSON
Writes {cfg: {bytes_per_candidate, src_sha, capture}} into OUT_JSON (merged);
bench.py reports roofline.traffic from it only while src_sha matches the
current kernel sources (bench.eval_src_sha)."""
import csv
import io
import json
import os
import subprocess
import sys

sys.path.insert(0, os.getcwd())
from bench import eval_src_sha  # noqa: E402

rep, cfg, K, out = sys.argv[1], sys.argv[2], int(sys.argv[3]), sys.argv[4]
raw = list(csv.reader(io.StringIO(subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"],
                                                 capture_output=True, text=True).stdout)))
h, units, vals = raw[0], raw[1], raw[2]
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
tot = 0.0
for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
    i = h.index(k)
    tot += float(vals[i].replace(",", "")) * scale[units[i]]
d = json.load(open(out)) if os.path.exists(out) else {}
d[cfg] = {"bytes_per_candidate": round(tot / K, 2), "src_sha": eval_src_sha(),
          "capture": f"ncu --set full, one eval2_kernel launch of K = {K}: dram read + write {tot:.0f} B"}
json.dump(d, open(out, "w"), indent=1)
print(cfg, d[cfg])
