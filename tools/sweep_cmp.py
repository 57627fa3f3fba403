"""Print two sweep JSON files side by side (GB/s encode / verify per config)."""
import json
import sys

a = {(r["dtype"], r["n"], r["nb"], r["lower_only"]): r for r in json.load(open(sys.argv[1]))}
b = {(r["dtype"], r["n"], r["nb"], r["lower_only"]): r for r in json.load(open(sys.argv[2]))}
for k in sorted(set(a) & set(b)):
    ra, rb = a[k], b[k]
    print(f"{k[0][-2:]} n={k[1]:6d} nb={k[2]:5d} {'L' if k[3] else 'F'}  enc {ra['encode_GBs']:7.0f} -> "
          f"{rb['encode_GBs']:7.0f}   ver {ra['verify_GBs']:7.0f} -> {rb['verify_GBs']:7.0f}")
