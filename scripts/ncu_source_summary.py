"""Per-role summary of an ncu source page (SASS view) of k_stream_tb_rt.

  python scripts/ncu_source_summary.py rep.ncu-rep > profiles/<name>_source.md

The SASS is cut at EXIT instructions; each segment is labelled by what it
contains (UTMALDG -> producer, STS -> intermediate stage, STG -> last stage, only
SYNCS retry loops -> wait loops). Reports stall samples, warp instructions,
shared wavefronts (actual / ideal) and the top stall reasons per segment, and the
instructions with the most samples.
"""
import collections
import csv
import subprocess
import sys


def main(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    kname, h, data = rows[0][1], rows[1], rows[2:]
    ix = {n: i for i, n in enumerate(h)}
    stalls = [c for c in h if c.startswith("stall_") and "Not Issued" not in c]
    num = lambda r, n: int(float(r[ix[n]] or 0))   # noqa: E731
    segs, cur = [], []
    for r in data:
        cur.append(r)
        if "EXIT" in r[1] and not r[1].strip().startswith("@"):
            segs.append(cur)
            cur = []
        elif "EXIT" in r[1]:
            segs.append(cur)
            cur = []
    if cur:
        segs.append(cur)
    tot = sum(num(r, "Warp Stall Sampling (All Samples)") for r in data)
    print(f"# ncu source page by role: `{kname[:110]}`\n")
    print(f"Report `{rep.split('/')[-1]}`; {tot} stall samples, {len(data)} SASS instructions. "
          "Segments end at EXIT instructions.\n")
    print("| segment | role | samples | % | warp instr | smem wavefronts | ideal | top stall reasons |")
    print("|---|---|---|---|---|---|---|---|")
    for k, sg in enumerate(segs):
        txt = " ".join(r[1] for r in sg)
        role = ("prologue (smem zero-fill, mbarrier init)" if "SYNCS.EXCH" in txt else "producer" if "UTMALDG" in txt else "last stage (STG)" if "STG" in txt else
                "intermediate stage (STS)" if "STS" in txt else "wait loops" if "NANOSLEEP" in txt else "setup")
        smp = sum(num(r, "Warp Stall Sampling (All Samples)") for r in sg)
        ex = sum(num(r, "Instructions Executed") for r in sg)
        wf = sum(num(r, "L1 Wavefronts Shared") for r in sg)
        wfi = sum(num(r, "L1 Wavefronts Shared Ideal") for r in sg)
        st = collections.Counter({c[6:]: sum(num(r, c) for r in sg) for c in stalls})
        top = ", ".join(f"{a} {b}" for a, b in st.most_common(4) if b)
        print(f"| {k} | {role} | {smp} | {100 * smp / max(tot, 1):.1f} | {ex} | {wf} | {wfi} | {top} |")
    print("\nInstructions with the most stall samples:\n")
    print("| # | SASS | samples | executed | top reason |")
    print("|---|---|---|---|---|")
    order = sorted(range(len(data)), key=lambda i: -num(data[i], "Warp Stall Sampling (All Samples)"))
    for i in order[:15]:
        r = data[i]
        st = max(stalls, key=lambda c: num(r, c))
        print(f"| {i} | `{r[1].strip()[:60]}` | {num(r, 'Warp Stall Sampling (All Samples)')} | "
              f"{num(r, 'Instructions Executed')} | {st[6:]} |")


if __name__ == "__main__":
    main(sys.argv[1])
