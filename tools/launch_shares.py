"""Per-kernel share of the C2 step from an ncu launch list (run here, no GPU needed).

usage: python tools/launch_shares.py gpurun_out/<tag>_launches.csv "<source note>" > profiles/<tag>_launch_shares.json

The CSV is the `ncu --metrics gpu__time_duration.sum --clock-control none --csv` pass over
`bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e`.  The bench's one separately timed
public-key encrypt launch (k_encrypt) is listed but excluded from the shares; in the two-launch
key-holder path the k_tc_exp<64> launches alternate stage 2 / decryption within a step.
"""
import collections
import csv
import json
import sys


def main():
    path, note = sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else ""
    rows = list(csv.reader(open(path)))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hi]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    scale = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0}
    tot, cnt = collections.Counter(), collections.Counter()
    seen64 = 0
    dag = any("k_tc_exp_dag" in r[ki] for r in rows[hi + 1:] if len(r) > ki)
    for r in rows[hi + 1:]:
        if len(r) <= vi:
            continue
        ms = float(r[vi].replace(",", "")) * scale[r[ui]]
        name = r[ki].split("(")[0].strip()
        if name.endswith("k_tc_exp<64>") and not dag:
            name += " (key-holder stage 2)" if seen64 % 2 == 0 else " (decryption)"
            seen64 += 1
        elif name.endswith("k_tc_exp<64>"):
            name += " (decryption)"
        tot[name] += ms
        cnt[name] += 1
    # the bench's separately timed public-key encryption (k_encrypt, or k_tc_exp<128> + its Philox fill
    # in the n^2 frame at 2048 bits) is not part of the key-holder C2 step
    def public(k):
        return "k_encrypt<" in k or "k_tc_exp<128>" in k or "k_tc_exp<(int)128>" in k

    step = sum(v for k, v in tot.items() if not public(k))
    out = {"source": note, "kernels": {}}
    for k, v in tot.most_common():
        pub = public(k)
        out["kernels"][k] = {"launches": cnt[k], "total_ms": round(v, 3),
                             "share_of_step_pct": None if pub else round(100 * v / step, 3)}
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
