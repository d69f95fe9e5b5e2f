"""Summarise a round's ncu evidence into profiles/:
  - the launch list (`--metrics gpu__time_duration.sum`, cold-cache, serialised): per-kernel share of a step
  - one `--set full` capture per hot kernel: duration, DRAM bytes, throughput, pipes, stalls
  - profiles/ncu_traffic.json: DRAM bytes per launch per bench family (bench.py roofline.traffic)
Usage: ncu_summary.py launches.csv out.md rep1.ncu-rep [rep2 ...]"""
import collections, csv, json, os, subprocess, sys

FAMILY = {"k_resblock": "sr_body", "k_recon_step": "recon", "k_uptail2": "sr_up", "k_conv_rot": "sr_head/end",
          "k_score": "score"}
UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6, "msecond": 1e-3,
        "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1,
        "second": 1}


def launches(path):
    rows = [r for r in csv.reader(open(path)) if len(r) > 10]
    h = rows[0]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    agg = collections.defaultdict(lambda: [0, 0.0])
    for r in rows[1:]:
        v = float(r[vi].replace(",", "")) * UNIT.get(r[ui], 1e-9 if r[ui] == "ns" else 1)
        n = r[ki].split("(")[0].replace("void ", "")
        agg[n][0] += 1
        agg[n][1] += v
    return agg


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    h, u, v = rows[0], rows[1], rows[2]
    d = {}
    for i, n in enumerate(h):
        try:
            d[n] = float(v[i].replace(",", "")) * UNIT.get(u[i], 1)
        except ValueError:
            d[n] = v[i]
    return d


def stalls(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    h = rows[1]
    agg = collections.Counter()
    for r in rows[2:]:
        if len(r) != len(h):
            continue
        for i, n in enumerate(h):
            if n.startswith("stall_") and "Not Issued" not in n and r[i] not in ("", "-"):
                agg[n[6:]] += float(r[i])
    t = sum(agg.values()) or 1
    return ", ".join(f"{k} {v / t:.0%}" for k, v in agg.most_common(6))


def main():
    lpath, md = sys.argv[1], sys.argv[2]
    reps = sys.argv[3:]
    agg = launches(lpath)
    tot = sum(a[1] for a in agg.values())
    lines = [f"# ncu summary ({os.path.basename(md).split("_")[0]}, c4 bench step; `tools/ncu_summary.py`)", "",
             f"Launch list: `{os.path.basename(lpath)}` -- `ncu --metrics gpu__time_duration.sum --clock-control none`, "
             "warm-up + 1 timed step of `bench.py` (cold-cache, serialised; shares, not absolute times, compare with "
             "the live CUDA-event breakdown in the bench JSON).", "",
             "| kernel | launches | ms (2 steps) | share |", "|---|---|---|---|"]
    for n, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
        lines.append(f"| `{n}` | {c} | {t * 1e3:.2f} | {t / tot:.1%} |")
    traffic = {}
    lines += ["", "## `--set full` captures (one launch each: SR kernels 16 jobs of 1280x720, recon one frame step of 64 streams)", "",
              "| kernel | duration ms | DRAM read GB | DRAM write GB | DRAM % peak | SM % | tensor pipe % | issue % | "
              "occupancy % | regs | top stalls |", "|---|---|---|---|---|---|---|---|---|---|---|"]
    for rep in reps:
        d = raw(rep)
        name = str(d.get("Kernel Name", os.path.basename(rep))).split("(")[0].replace("void ", "").replace("ns::", "")
        base = name.split("<")[0]
        rd, wr = d.get("dram__bytes_read.sum", 0.0), d.get("dram__bytes_write.sum", 0.0)
        fam = FAMILY.get(base)
        if fam:
            traffic[fam] = rd + wr
        g = lambda k: d.get(k, float("nan"))
        lines.append(
            f"| `{name}` | {g('gpu__time_duration.sum') * 1e3:.3f} | {rd / 1e9:.3f} | {wr / 1e9:.3f} | "
            f"{g('gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed'):.1f} | "
            f"{g('sm__throughput.avg.pct_of_peak_sustained_elapsed'):.1f} | "
            f"{g('sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active'):.1f} | "
            f"{g('sm__inst_issued.avg.pct_of_peak_sustained_active'):.1f} | "
            f"{g('sm__warps_active.avg.pct_of_peak_sustained_active'):.1f} | {g('launch__registers_per_thread'):.0f} | "
            f"{stalls(rep)} |")
    open(md, "w").write("\n".join(lines) + "\n")
    json.dump(traffic, open(os.path.join(os.path.dirname(md), "ncu_traffic.json"), "w"), indent=1)
    print("\n".join(lines))
    print(traffic)


if __name__ == "__main__":
    main()
