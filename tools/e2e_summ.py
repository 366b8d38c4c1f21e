"""One line per run of tools/e2e_breakdown.py output blocks ("<label>" line, then the JSON line):
label, host-to-host interactions/s (zero-copy in + out), wall ms.  python tools/e2e_summ.py file"""
import json
import sys

k = None
for ln in open(sys.argv[1]):
    ln = ln.strip()
    if ln.startswith("{"):
        d = json.loads(ln)
        print(k, d["1"]["wall_e12"], d["1"]["wall_ms"])
    elif ln:
        k = ln
