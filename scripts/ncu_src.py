"""Per-source-line shares (instructions executed, warp-stall samples) of the kernels in
an ncu report, from the `--print-source cuda,sass` page (needs -lineinfo and
--import-source on at capture).  usage: ncu_src.py <report> [kernel-regex] [top]"""
import csv
import subprocess
import sys
from collections import defaultdict


def main(rep, kre=None, top=40):
    args = ["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"]
    if kre:
        args += ["-k", f"regex:{kre}"]
    out = subprocess.run(args, capture_output=True, text=True).stdout
    E, S, txt = defaultdict(int), defaultdict(int), {}
    stall = defaultdict(lambda: defaultdict(int))
    f = fn = None
    hdr = None
    for r in csv.reader(out.splitlines()):
        if not r:
            continue
        if r[0] == "File Path":
            f = r[1].split("/")[-1]
            continue
        if r[0] == "Function Name":
            fn = r[1]
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or not r[0].isdigit():
            continue
        k = (f, int(r[0]))
        ie, iss = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)")
        try:
            E[k] += int(r[ie] or 0)
            S[k] += int(r[iss] or 0)
        except ValueError:
            continue
        txt[k] = r[1]
        for j, c in enumerate(hdr):
            if c.startswith("stall_") and "Not Issued" not in c:
                try:
                    stall[k][c[6:]] += int(r[j] or 0)
                except ValueError:
                    pass
    te, ts = sum(E.values()) or 1, sum(S.values()) or 1
    print(f"{fn}: {te} warp instructions, {ts} stall samples")
    for k, v in sorted(E.items(), key=lambda x: -(x[1] / te + S[x[0]] / ts))[:top]:
        st = sorted(stall[k].items(), key=lambda x: -x[1])[:2]
        sts = " ".join(f"{a}:{100 * b / max(S[k], 1):.0f}%" for a, b in st if b)
        print(f"{100 * v / te:5.1f}% inst {100 * S[k] / ts:5.1f}% smp  {k[0]}:{k[1]:<5} {txt[k].strip()[:70]:70s} {sts}")


if __name__ == "__main__":
    a = sys.argv
    main(a[1], a[2] if len(a) > 2 and a[2] else None, int(a[3]) if len(a) > 3 else 40)
