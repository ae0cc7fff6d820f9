"""Summarise an ncu capture (--set full) into profiles/<name>.md and record the dominant
kernel's DRAM traffic per launch in profiles/traffic.json (read by bench.py)."""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
METRICS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
           "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
           "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
           "smsp__warps_eligible.avg.per_cycle_active", "launch__registers_per_thread", "launch__grid_size",
           "launch__block_size", "launch__shared_mem_per_block_dynamic", "smsp__inst_executed.sum",
           "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "lts__t_sector_hit_rate.pct"]


def ncu_csv(rep, *args):
    out = subprocess.run(["ncu", "-i", rep, "--csv", *args], capture_output=True, text=True).stdout
    lines = [l for l in out.splitlines() if l.startswith('"')]
    return list(csv.reader(io.StringIO("\n".join(lines))))


def bytes_of(v, unit):
    f = float(v.replace(",", ""))
    return f * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(unit, 1)


def main(rep, name, cfg, alg_bytes=None, note=""):
    raw = ncu_csv(rep, "--page", "raw")
    h, units = raw[0], raw[1]
    row = raw[2]
    get = lambda k: (row[h.index(k)], units[h.index(k)]) if k in h else (None, None)
    kname = row[h.index("Kernel Name")] if "Kernel Name" in h else "?"
    lines = [f"# ncu summary: {name}", "", f"kernel: `{kname}`", "", f"capture: `{os.path.basename(rep)}` "
             "(`ncu --set full --clock-control none --import-source on`, one launch, scripts/gpu_prof.sh)", ""]
    if note:
        lines += [note, ""]
    lines += ["| metric | value | unit |", "|---|---|---|"]
    for k in METRICS:
        v, u = get(k)
        if v is not None:
            lines.append(f"| {k} | {v} | {u} |")
    rd, ru = get("dram__bytes_read.sum")
    wr, wu = get("dram__bytes_write.sum")
    traffic = bytes_of(rd, ru) + bytes_of(wr, wu)
    lines += ["", f"DRAM traffic per launch: {traffic / 1e9:.3f} GB"]
    if alg_bytes:
        lines.append(f"algorithmic bytes per launch: {alg_bytes / 1e9:.3f} GB (traffic / algorithmic = {traffic / alg_bytes:.3f})")
    # stall reasons from the source page
    src = ncu_csv(rep, "--page", "source", "--print-source", "sass")
    if len(src) > 2:
        sh = src[1] if "Source" in src[1] else src[0]
        data = src[2:] if "Source" in src[1] else src[1:]
        cols = [c for c in sh if c.startswith("stall_") and "Not Issued" not in c]
        tot = {c: 0 for c in cols}
        for r in data:
            for c in cols:
                try:
                    tot[c] += int(r[sh.index(c)] or 0)
                except (ValueError, IndexError):
                    pass
        s = sum(tot.values()) or 1
        lines += ["", "warp stall samples (share of all samples):", "", "| reason | share |", "|---|---|"]
        for c, v in sorted(tot.items(), key=lambda x: -x[1])[:10]:
            lines.append(f"| {c[6:]} | {100 * v / s:.1f}% |")
    outdir = os.environ.get("RW_PROFILE_DIR", os.path.join(ROOT, "profiles"))
    os.makedirs(outdir, exist_ok=True)
    with open(os.path.join(outdir, f"{name}.md"), "w") as f:
        f.write("\n".join(lines) + "\n")
    tj = os.path.join(outdir, "traffic.json")
    t = json.load(open(tj)) if os.path.exists(tj) else {}
    t[cfg] = traffic
    json.dump(t, open(tj, "w"), indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], sys.argv[3], float(sys.argv[4]) if len(sys.argv) > 4 else None,
         sys.argv[5] if len(sys.argv) > 5 else "")
