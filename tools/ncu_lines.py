"""Aggregate an ncu source page (--print-source cuda,sass, CSV) to source lines: warp-stall samples and
warp instructions executed per line, top N (run here, no GPU needed).
    ncu -i rep.ncu-rep --page source --csv --print-source cuda,sass > src.csv
    python tools/ncu_lines.py src.csv [N]"""
import collections
import csv
import os
import sys

path = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
samples, insts, text = collections.Counter(), collections.Counter(), {}
ops = collections.defaultdict(collections.Counter)
cur_file, cur = None, None
for row in csv.reader(open(path)):
    if not row:
        continue
    if row[0] == "File Path":
        cur_file = os.path.basename(row[1])
        continue
    if row[0] in ("Function Name", "Line No"):
        continue
    if row[0]:
        cur = (cur_file, int(row[0]))
        text[cur] = row[1].strip()
        continue
    if len(row) > 7 and row[2].startswith("0x") and cur:
        try:
            s, n = int(row[4]), int(row[7])
        except ValueError:
            continue
        samples[cur] += s
        insts[cur] += n
        ops[cur][row[3].split()[0] if row[3].split() else "?"] += n
tot_s, tot_i = sum(samples.values()) or 1, sum(insts.values()) or 1
print(f"total samples {tot_s}, warp instructions {tot_i}")
for key, s in samples.most_common(top):
    mix = ",".join(f"{o}:{c * 100 // max(insts[key], 1)}" for o, c in ops[key].most_common(3))
    print(f"{100 * s / tot_s:5.1f}% smp {100 * insts[key] / tot_i:5.1f}% ins  {key[0]}:{key[1]:<5} {text[key][:90]}  [{mix}]")
