"""Summarise ncu captures (gpurun_out/full_<cfg>.ncu-rep, launches_c3.csv) into
profiles/ncu_summary.json (read by bench.py for roofline.traffic) and a
markdown digest profiles/<round>_summary.md.

usage: python tools/make_profiles.py r01 [C3 C2 C4]
"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.environ.get("NCU_DIR") or os.path.join(ROOT, "gpurun_out")  # where full_<cfg>.ncu-rep live
PROF = os.environ.get("PROF_DIR") or os.path.join(ROOT, "profiles")  # the GPU box writes into gpurun_out/

KERNELS = ("gbtrf_tpm_kernel", "gbtrf_cols_kernel", "gbtrf_rows_kernel", "gbtrf_window_kernel", "gbtrf_wide_kernel", "gbtrf_tc_kernel", "gbtrf_generic_kernel",
           "gbtrs_window_kernel", "gbtrs_bwd_kernel", "gbtrs_rows_kernel", "gbtrs_generic_kernel", "gbtrs_t_generic_kernel",
           "gbtrs_blk_kernel", "gbtrs_t_kernel")
KEYS = {
    "duration_us": ("gpu__time_duration.sum", 1e-3),
    "dram_bytes_read": ("dram__bytes_read.sum", 1.0),
    "dram_bytes_write": ("dram__bytes_write.sum", 1.0),
    "dram_throughput_pct": ("dram__throughput.avg.pct_of_peak_sustained_elapsed", 1.0),
    "inst_executed": ("smsp__inst_executed.sum", 1.0),
    "issue_active_pct": ("smsp__issue_active.avg.pct_of_peak_sustained_active", 1.0),
    "fp64_pipe_pct": ("sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active", 1.0),
    "warps_active_pct": ("sm__warps_active.avg.pct_of_peak_sustained_active", 1.0),
    "registers": ("launch__registers_per_thread", 1.0),
    "smem_bank_conflicts": ("l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", 1.0),
    "lsu_wavefronts_pct": ("l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed", 1.0),
}
UNIT_SCALE = {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1.0, "ms": 1e3, "us": 1.0, "usecond": 1.0,
              "msecond": 1e3, "nsecond": 1e-3, "ns": 1e-3}


def raw(rep):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(txt)))
    return r[0], r[1], r[2:]


def summarise(rep):
    hdr, units, rows = raw(rep)
    out = {}
    for row in rows:
        name = row[hdr.index("Kernel Name")]
        kern = next((k for k in KERNELS if k in name), name)
        d = {"kernel_full": name}
        for k, (m, _) in KEYS.items():
            if m in hdr:
                i = hdr.index(m)
                try:
                    v = float(row[i])
                except ValueError:
                    continue
                u = units[i]
                if k == "duration_us":
                    v = v * UNIT_SCALE.get(u, 1.0)
                elif k.startswith("dram_bytes"):
                    v = v * UNIT_SCALE.get(u, 1.0)
                d[k] = v
        st = []
        for h, v in zip(hdr, row):
            if h.startswith("smsp__pcsamp_warps_issue_stalled") and not h.endswith("not_issued"):
                try:
                    st.append((float(v), h.replace("smsp__pcsamp_warps_issue_stalled_", "")))
                except ValueError:
                    pass
        tot = sum(x for x, _ in st) or 1.0
        d["top_stalls_pct"] = {h: round(100 * x / tot, 1) for x, h in sorted(st, reverse=True)[:6]}
        out[kern] = d
    return out


def launches(csvpath):
    if not os.path.exists(csvpath):
        return None
    txt = open(csvpath).read()
    txt = txt[txt.index('"ID"'):] if '"ID"' in txt else txt
    r = list(csv.DictReader(io.StringIO(txt)))
    agg = {}
    for row in r:
        nm = row.get("Kernel Name", "")
        key = next((k for k in KERNELS if k in nm), nm[:60])
        try:
            v = float(row["Metric Value"])
        except (KeyError, ValueError):
            continue
        scale = UNIT_SCALE.get(row.get("Metric Unit", "ns"), 1e-3)  # -> us
        a = agg.setdefault(key, [0, 0.0])
        a[0] += 1
        a[1] += v * scale
    return agg


def main():
    rnd = sys.argv[1] if len(sys.argv) > 1 else "r01"
    cfgs = sys.argv[2:] or ["C3", "C2", "C4"]
    os.makedirs(PROF, exist_ok=True)
    jpath = os.path.join(PROF, "ncu_summary.json")
    summary = json.load(open(jpath)) if os.path.exists(jpath) else {}
    md = [f"# ncu summary, round {rnd}", "",
          "Captured with `ncu --set full --clock-control none --import-source on -k regex:gbtr` on one B200",
          "(`tools/prof_step.py <cfg>`: one dgbtrfs step -- the library's plan -- at the BASELINE config;",
          "C5W = C5's (32,32) band at n = 512, batch 4,000). ncu times are",
          "cold-cache and serialised; bench.py numbers come from CUDA events without a profiler.", ""]
    for c in cfgs:
        rep = os.path.join(OUT, f"full_{c}.ncu-rep")
        if not os.path.exists(rep):
            continue
        s = summarise(rep)
        summary[c] = s
        md.append(f"## {c}")
        md.append("")
        md.append("| kernel | us | DRAM read GB | DRAM write GB | DRAM GB/s | issue % | FP64 pipe % | regs | top stalls |")
        md.append("|---|---|---|---|---|---|---|---|---|")
        for k, d in s.items():
            md.append(f"| {k} | {d.get('duration_us', 0):.1f} | {d.get('dram_bytes_read', 0)/1e9:.3f} | "
                      f"{d.get('dram_bytes_write', 0)/1e9:.3f} | "
                      f"{(d.get('dram_bytes_read', 0) + d.get('dram_bytes_write', 0)) / max(d.get('duration_us', 1), 1e-9) / 1e3:.0f} | "
                      f"{d.get('issue_active_pct', 0):.1f} | {d.get('fp64_pipe_pct', 0):.1f} | {d.get('registers', 0):.0f} | "
                      + ", ".join(f"{h} {p}%" for h, p in d["top_stalls_pct"].items()) + " |")
        md.append("")
    la = launches(os.path.join(OUT, "launches_c3.csv"))
    if la:
        tot = sum(v[1] for v in la.values())
        md.append("## Launch list of `bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-cpu` (C3)")
        md.append("")
        md.append("| kernel | launches | total us | share of GPU time |")
        md.append("|---|---|---|---|")
        for k, (n, t) in sorted(la.items(), key=lambda x: -x[1][1]):
            md.append(f"| {k} | {n} | {t:.1f} | {100 * t / tot:.1f}% |")
        md.append("")
    json.dump(summary, open(jpath, "w"), indent=1)
    open(os.path.join(PROF, f"{rnd}_summary.md"), "w").write("\n".join(md) + "\n")
    print("\n".join(md))


if __name__ == "__main__":
    main()
