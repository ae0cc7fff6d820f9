"""Per-source-line instruction and stall-sample shares of one kernel in an ncu report.
usage: ncu_lines.py <report> <kernel-regex> <lib.so> <mangled-name-substring> [section] [top]
The .so must be the exact binary that was profiled (line info from nvdisasm -g)."""
import csv, os, re, subprocess, sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def linemap(lib, pat):
    d = "/tmp/_ncu_lines_cubin"
    os.makedirs(d, exist_ok=True)
    subprocess.run(f"cd {d} && rm -f *.cubin && cuobjdump -xelf all {lib} > /dev/null 2>&1", shell=True)
    lines = []
    for cub in sorted(os.listdir(d)):
        txt = subprocess.run(["nvdisasm", "-g", "-c", os.path.join(d, cub)], capture_output=True, text=True).stdout.splitlines()
        st = [i for i, l in enumerate(txt) if l.startswith("//----") and pat in l]
        if not st:
            continue
        st = st[0]
        en = [i for i, l in enumerate(txt) if i > st + 5 and l.startswith("//---------------------")]
        en = en[0] if en else len(txt)
        cur = None
        for l in txt[st:en]:
            m = re.search(r'## File "(.*?)", line (\d+)', l)
            if m:
                cur = (m.group(1).split("/")[-1], int(m.group(2)))
                continue
            if re.match(r"\s+/\*([0-9a-f]{4,})\*/\s+", l):
                lines.append(cur)
        break
    return lines


def main(rep, kre, lib, pat, section=0, top=30):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass", "-k", f"regex:{kre}"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    idx = [i for i, r in enumerate(rows) if r and r[0] == "Kernel Name"]
    a = idx[section]
    b = idx[section + 1] if section + 1 < len(idx) else len(rows)
    h, data = rows[a + 1], rows[a + 2:b]
    lm = linemap(lib, pat)
    if len(lm) != len(data):
        print(f"warning: {len(lm)} mapped instructions vs {len(data)} profiled")
    iss, iex = h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
    E, S = defaultdict(int), defaultdict(int)
    for i, r in enumerate(data):
        k = lm[i] if i < len(lm) else None
        E[k] += int(r[iex] or 0)
        S[k] += int(r[iss] or 0)
    te, ts = sum(E.values()) or 1, sum(S.values()) or 1
    src = {}
    for f in ["kernels.cu", "chain.cuh", "ptx.cuh", "dist_kernels.cu"]:
        pth = os.path.join(ROOT, "paper_conf_micro_wudcy12_b200", "csrc", f)
        if os.path.exists(pth):
            src[f] = open(pth).read().splitlines()
    print(f"{rows[a][1][:100]}: {te} instructions, {ts} samples")
    for k, v in sorted(E.items(), key=lambda x: -x[1])[:top]:
        s = src[k[0]][k[1] - 1].strip()[:80] if k and k[0] in src and k[1] <= len(src[k[0]]) else ""
        print(f"{100 * v / te:5.1f}% inst {100 * S[k] / ts:5.1f}% smp  {k[0] if k else '?'}:{k[1] if k else ''}  {s}")


if __name__ == "__main__":
    a = sys.argv
    main(a[1], a[2], a[3], a[4], int(a[5]) if len(a) > 5 else 0, int(a[6]) if len(a) > 6 else 30)
