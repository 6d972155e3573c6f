#!/usr/bin/env python
"""Stall reasons and instruction mix of one kernel from an `ncu --page source --csv` export.

    python scripts/ncu_stalls.py SOURCE_CSV OUT_JSON "kernel description"
"""
import collections
import csv
import json
import sys


def main(src, out, what):
    rows = list(csv.reader(open(src)))
    hdr, data = rows[1], rows[2:]
    isrc, iex = hdr.index("Source"), hdr.index("Instructions Executed")
    idx = {h: hdr.index(h) for h in hdr if h.startswith("stall_") and "Not Issued" not in h}
    stalls, ops, n = collections.Counter(), collections.Counter(), 0
    for r in data:
        s = r[isrc].strip()
        if not s:
            continue
        t = s.split()
        op = (t[1] if t[0].startswith("@") else t[0]).split(".")[0]
        try:
            ops[op] += int(r[iex])
            n += int(r[iex])
        except ValueError:
            pass
        for k, i in idx.items():
            try:
                stalls[k] += int(r[i])
            except ValueError:
                pass
    tot = sum(stalls.values())
    res = {"kernel": what, "warp_instructions": n,
           "stall_share_pct": {k: round(100 * v / tot, 1) for k, v in stalls.most_common() if v},
           "instruction_mix_pct": {k: round(100 * v / n, 1) for k, v in ops.most_common(16)}}
    json.dump(res, open(out, "w"), indent=1)
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main(*sys.argv[1:4])
