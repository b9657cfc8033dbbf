"""Summarise ncu outputs of one GPU session into profiles/ (test-side tool, runs here without a GPU).

  python tools/ncu_summary.py gpurun_out/r01b profiles/r01b

Reads (when present): launches_n32768.csv (gpu__time_duration per launch), traffic_n32768.csv (DRAM/L2
bytes per launch), prof_*.ncu-rep (--set full captures).  Writes <out>_launches.json (per-kernel-class
share of the step, launch counts), <out>_traffic.json (per-class DRAM bytes per launch; also merged into
profiles/ncu_traffic.json for bench.py's roofline.traffic) and <out>_full.json (key counters per capture).
Kernel classes follow the DBBR/BC stage names: a ws_kernel<128,64,...,0> launch right after the W = Y T
launch of a panel is the SYMM (second ws_kernel after each panel_reg_kernel), ws_kernel<128,128,...> is the
syr2k, panel_* the panel QR, bc_* the bulge chase."""
import csv
import json
import os
import subprocess
import sys
from collections import defaultdict


def read_ncu_csv(path):
    rows = []
    with open(path) as f:
        lines = [ln for ln in f if ln.startswith('"')]
    rd = csv.reader(lines)
    hdr = next(rd, None)
    if hdr is None:
        return rows
    for r in rd:
        rows.append(dict(zip(hdr, r)))
    return rows


def per_launch(rows):
    """{launch id: {"name": ..., metric: value}} from a --csv metrics log."""
    out = {}
    for r in rows:
        i = int(r["ID"])
        d = out.setdefault(i, {"name": r["Kernel Name"]})
        try:
            d[r["Metric Name"]] = float(r["Metric Value"].replace(",", ""))
        except ValueError:
            d[r["Metric Name"]] = float("nan")
    return [out[i] for i in sorted(out)]


def classify(launches):
    """Assign each launch a stage class.  Per panel (the launches between two panel_* launches): the first
    ws_kernel<128, 64, 4, 2, 0> is W = Y T, the longest one is the SYMM (with the folded corrections) and the
    ws_reduce_kernel right after it belongs to it, ws_kernel<.., 1, 0> (B op T) is the next-panel update, the other
    skinny launches (the stacked U, S, Z and their reductions) are the Z tail; ws_kernel<128, 128, ...> is the syr2k,
    bc_* / band_* the chase."""
    cls = [None] * len(launches)
    group = []

    def flush():
        ws0 = [i for i in group if "ws_kernel<128, 64, 4, 2, 0" in launches[i]["name"]]
        if not ws0:
            return
        w_i = ws0[0]
        rest = ws0[1:]
        s_i = max(rest, key=lambda i: launches[i].get("gpu__time_duration.sum", 0.0)) if rest else None
        for i in group:
            nm = launches[i]["name"]
            if i == w_i:
                cls[i] = "wy"
            elif i == s_i:
                cls[i] = "symm"
            elif "ws_kernel<128, 64, 4, 2, 1" in nm:
                cls[i] = "next_panel"
            elif "ws_reduce_kernel" in nm and s_i is not None and i == s_i + 1:
                cls[i] = "symm"
            else:
                cls[i] = "zy"

    for i, d in enumerate(launches):
        nm = d["name"]
        if "panel_" in nm:
            flush()
            group = []
            cls[i] = "panel_qr"
        elif "ws_kernel<128, 128" in nm:
            flush()
            group = []
            cls[i] = "syr2k"
        elif "bc_" in nm or "band_" in nm:
            cls[i] = "bulge_chase"
        elif "ws_" in nm or "gemm_kernel" in nm or "reduce_partials" in nm:
            group.append(i)
        elif "trid::" in nm:
            cls[i] = "other_trid"
        else:
            cls[i] = "torch"
    flush()
    return [c or "other_trid" for c in cls]


def summarize_launches(path):
    L = per_launch(read_ncu_csv(path))
    cls = classify(L)
    tot = defaultdict(float)
    cnt = defaultdict(int)
    for d, c in zip(L, cls):
        t = d.get("gpu__time_duration.sum", float("nan"))
        if t == t:
            tot[c] += t
            cnt[c] += 1
    step = sum(v for c, v in tot.items() if c != "torch")
    return {"source": os.path.basename(path), "note": "ncu serialised, cold-cache per-launch times: compare SHARES",
            "classes": {c: {"ms": round(tot[c] / 1e6, 3), "launches": cnt[c],
                            "share_of_trid": round(tot[c] / step, 4) if c != "torch" and step else None}
                        for c in sorted(tot)}}, L, cls


def summarize_traffic(path):
    L = per_launch(read_ncu_csv(path))
    cls = classify(L)
    agg = defaultdict(lambda: defaultdict(float))
    for d, c in zip(L, cls):
        a = agg[c]
        a["launches"] += 1
        for k in ("dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum", "gpu__time_duration.sum"):
            v = d.get(k, float("nan"))
            if v == v:
                a[k] += v
    out = {}
    for c, a in agg.items():
        n = max(a["launches"], 1)
        out[c] = {"launches": int(a["launches"]),
                  "dram_bytes_per_launch": (a["dram__bytes_read.sum"] + a["dram__bytes_write.sum"]) / n,
                  "dram_read_per_launch": a["dram__bytes_read.sum"] / n,
                  "dram_write_per_launch": a["dram__bytes_write.sum"] / n,
                  "l2_bytes_per_launch": a["lts__t_bytes.sum"] / n}
    return out


KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_sectors.sum",
        "sm__inst_executed_pipe_tensor_subpipe_dmma.avg.pct_of_peak_sustained_active",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__issue_active.avg.per_cycle_active",
        "launch__grid_size", "launch__block_size", "launch__shared_mem_per_block_dynamic"]
STALLS = "smsp__average_warps_issue_stalled_"


def summarize_full(rep):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    lines = [ln for ln in raw.splitlines() if ln.startswith('"')]
    rd = csv.reader(lines)
    hdr = next(rd, None)
    if hdr is None:
        return []
    units = next(rd)
    res = []
    for r in rd:
        d = dict(zip(hdr, r))
        u = dict(zip(hdr, units))
        item = {"kernel": d.get("Kernel Name")}
        for k in KEYS:
            if k in d:
                item[k] = f"{d[k]} {u.get(k, '')}".strip()
        st = {k[len(STALLS):].replace("_per_issue_active.ratio", ""): float(d[k]) for k in hdr
              if k.startswith(STALLS) and k.endswith("_per_issue_active.ratio") and d[k] not in ("", "n/a")}
        item["top_stalls_per_issue"] = dict(sorted(st.items(), key=lambda kv: -kv[1])[:6])
        res.append(item)
    return res


def main():
    src, out = sys.argv[1], sys.argv[2]
    os.makedirs(os.path.dirname(out) or ".", exist_ok=True)
    lp = os.path.join(src, "launches_n32768.csv")
    if os.path.exists(lp):
        s, _, _ = summarize_launches(lp)
        json.dump(s, open(out + "_launches.json", "w"), indent=1)
        print(json.dumps(s, indent=1))
    tp = os.path.join(src, "traffic_n32768.csv")
    if os.path.exists(tp) and read_ncu_csv(tp):
        t = summarize_traffic(tp)
        json.dump(t, open(out + "_traffic.json", "w"), indent=1)
        # per-class averages over every launch of the class (incl. its split-K reductions) stay in <out>_traffic.json;
        # profiles/ncu_traffic.json (bench.py's roofline.traffic) holds per-kernel figures from --set full captures,
        # curated by hand with their provenance
        print(json.dumps(t, indent=1))
    full = {}
    for f in sorted(os.listdir(src)):
        if f.startswith("prof_") and f.endswith(".ncu-rep"):
            try:
                full[f[5:-8]] = summarize_full(os.path.join(src, f))
            except Exception as ex:  # noqa: BLE001
                full[f[5:-8]] = {"error": str(ex)}
    if full:
        json.dump(full, open(out + "_full.json", "w"), indent=1)
        print(json.dumps(full, indent=1)[:4000])


if __name__ == "__main__":
    main()
