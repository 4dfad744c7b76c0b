"""Summarise ncu captures from gpurun_out/ into committed profiles/ files.

  python tools/make_profiles.py ROUND   (e.g. r1)

Reads gpurun_out/launches_c{2,3}.csv (ncu --metrics gpu__time_duration.sum,dram__bytes_*: every
launch of a short bench.py run, cold-cache and serialised) and gpurun_out/full_c{2,3}_*.ncu-rep
(ncu --set full of each kernel), writes profiles/ROUND_launches_cN.txt, profiles/ROUND_full_cN_K.txt
and profiles/ncu_traffic.json (per-kernel DRAM bytes per launch, read by bench.py's roofline).
"""
import collections
import csv
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.environ.get("PROF_OUT") or os.path.join(ROOT, "profiles")  # PROF_OUT: e.g. gpurun_out/prof on the box
def kname(full):
    """Map an ncu kernel name to the bench.py stage name (template args decide the variant)."""
    import re
    m = re.search(r"(tc_gemm1|tc_gemm2)<([^>]*)>", full)
    if m:
        a = [x.strip() for x in m.group(2).split(",")]
        flags = [x in ("true", "1", "(bool)1") for x in a[2:]]
        if m.group(1) == "tc_gemm1":  # <D, T, LS, PAIR, IRT>
            if not (flags and flags[0]):
                return "gemm1_plain"
            return "gemm1_ls_ir" if len(flags) > 2 and flags[2] else "gemm1_ls"
        if flags and flags[0]:  # <D, T, GS, FI, RS>
            if len(flags) > 2 and flags[2]:
                return "gs_gemm2"  # default path: (m, 1/d) from GEMM1
            return "gs_gemm2_fused_ir" if len(flags) > 1 and flags[1] else "gs_gemm2_rprime"
        return "gemm2_plain"
    if "tc_fused" in full:
        return "sr_layer_one_kernel"
    if "sched_upload" in full:
        return "sched_upload"
    if "tc_bwd_kv" in full:
        return "bwd_dkdv"
    for k, v in (("ir_kernel", "ir"), ("row_softmax", "softmax"), ("sd_ls_kernel", "sd_ls"),
                 ("sd_gs_kernel", "sd_gs"), ("tc_bwd_ds", "bwd_ds"), ("bwd_prep", "bwd_prep")):
        if k in full:
            return v
    return None


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hdr]
    agg = collections.defaultdict(lambda: collections.defaultdict(list))
    order = []
    for r in rows[hdr + 1:]:
        if len(r) != len(h):
            continue
        d = dict(zip(h, r))
        n = kname(d["Kernel Name"]) or ("other:" + d["Kernel Name"][:40])
        if n not in order:
            order.append(n)
        agg[n][d["Metric Name"]].append(float(d["Metric Value"].replace(",", "")))
    return order, agg


def main(rnd):
    os.makedirs(PROF, exist_ok=True)
    tp = os.path.join(PROF, "ncu_traffic.json")
    traffic = json.load(open(tp)) if os.path.exists(tp) else {}  # configs not re-profiled keep their entry
    for c in (2, 3, 4, 5, 6):
        p = os.path.join(OUT, f"launches_c{c}.csv")
        if not os.path.exists(p):
            continue
        order, agg = launches(p)
        lines = [f"# ncu launch list, bench.py --config {c} (cold-cache, serialised launches; compare SHARES)",
                 f"{'kernel':28s} {'launches':>8s} {'mean us':>10s} {'DRAM rd MB':>11s} {'DRAM wr MB':>11s}"]
        ours = {}
        for n in order:
            m = agg[n]
            t = sum(m["gpu__time_duration.sum"]) / len(m["gpu__time_duration.sum"])
            rd = sum(m["dram__bytes_read.sum"]) / len(m["dram__bytes_read.sum"])
            wr = sum(m["dram__bytes_write.sum"]) / len(m["dram__bytes_write.sum"])
            unit = 1.0
            lines.append(f"{n:28s} {len(m['gpu__time_duration.sum']):8d} {t / 1e3 * unit:10.2f} {rd / 1e6:11.2f} {wr / 1e6:11.2f}")
            if not n.startswith("other"):
                ours[n] = (t, rd + wr)
        rec = [k for k in ("sr_layer_one_kernel",) if k in ours]  # default path: one launch (+ schedule upload)
        up = ours.get("sched_upload")
        two = [k for k in ("gemm1_ls_ir", "gs_gemm2") if k in ours]  # SR_TWO_KERNELS
        unf = [k for k in ("gemm1_plain", "softmax", "gemm2_plain") if k in ours]
        tr = sum(ours[k][0] for k in rec)
        lines.append("")
        lines.append("recomposed layer (default, one launch): " + ", ".join(f"{k} {ours[k][0] / 1e3:.2f} us" for k in rec)
                     + (f" (+ schedule upload {up[0] / 1e3:.2f} us per launch, "
                        f"{ours['sr_layer_one_kernel'][0] / (ours['sr_layer_one_kernel'][0] + up[0]):.1%} kernel share)"
                        if up and rec else ""))
        if len(two) == 2:
            t2 = sum(ours[k][0] for k in two)
            lines.append("two-kernel variant shares: " + ", ".join(f"{k} {ours[k][0] / t2:.1%}" for k in two))
        tu = sum(ours[k][0] for k in unf) if unf else 0
        if unf:
            lines.append("unfused layer shares:    " + ", ".join(f"{k} {ours[k][0] / tu:.1%}" for k in unf))
        irk = [k for k in ("gemm1_ls", "ir", "gs_gemm2_rprime") if k in ours]
        if len(irk) == 3:
            tk = sum(ours[k][0] for k in irk)
            lines.append("IR-kernel (paper layout) shares: " + ", ".join(f"{k} {ours[k][0] / tk:.1%}" for k in irk))
        fir = [k for k in ("gemm1_ls", "gs_gemm2_fused_ir") if k in ours]
        if len(fir) == 2:
            tf = sum(ours[k][0] for k in fir)
            lines.append("fused-IR variant shares: " + ", ".join(f"{k} {ours[k][0] / tf:.1%}" for k in fir))
        sd = [k for k in ("gemm1_plain", "sd_ls", "ir", "sd_gs", "gemm2_plain") if k in ours]
        if len(sd) == 5:
            ts = sum(ours[k][0] for k in sd)
            lines.append("SD variant shares:       " + ", ".join(f"{k} {ours[k][0] / ts:.1%}" for k in sd))
        e = {f"{k}_dram_bytes": int(ours[k][1]) for k in ours}
        e["recomposed_dram_bytes"] = int(sum(ours[k][1] for k in rec))
        if len(irk) == 3:
            e["ir_kernel_dram_bytes"] = int(sum(ours[k][1] for k in irk))
        if unf:
            e["unfused_dram_bytes"] = int(sum(ours[k][1] for k in unf))
        lines.append(f"DRAM bytes per layer (cold, per-kernel sum): recomposed {e['recomposed_dram_bytes'] / 1e6:.1f} MB"
                     + (f", unfused {e['unfused_dram_bytes'] / 1e6:.1f} MB" if unf else ""))
        pt = os.path.join(OUT, f"launches_train_c{c}.csv")  # ncu of tools/run_layer.py C train
        if os.path.exists(pt):
            o2, a2 = launches(pt)
            lines += ["", f"# training step (tools/run_layer.py {c} train): forward + backward, cold-cache launches",
                      f"{'kernel':28s} {'launches':>8s} {'mean us':>10s} {'DRAM rd MB':>11s} {'DRAM wr MB':>11s}"]
            bw = {}
            for n in o2:
                m = a2[n]
                t = sum(m["gpu__time_duration.sum"]) / len(m["gpu__time_duration.sum"])
                rd = sum(m["dram__bytes_read.sum"]) / len(m["dram__bytes_read.sum"])
                wr = sum(m["dram__bytes_write.sum"]) / len(m["dram__bytes_write.sum"])
                nm = "bwd_dq (gemm2_plain)" if n == "gemm2_plain" else n
                lines.append(f"{nm:28s} {len(m['gpu__time_duration.sum']):8d} {t / 1e3:10.2f} {rd / 1e6:11.2f} {wr / 1e6:11.2f}")
                if n in ("bwd_prep", "bwd_ds", "gemm2_plain", "bwd_dkdv"):
                    bw["bwd_dq" if n == "gemm2_plain" else n] = (t, rd + wr)
            if bw:
                tb = sum(v[0] for v in bw.values())
                lines.append("backward shares: " + ", ".join(f"{k} {v[0] / tb:.1%}" for k, v in bw.items()))
                lines.append(f"backward DRAM bytes (cold, per-kernel sum): {sum(v[1] for v in bw.values()) / 1e6:.1f} MB")
                e.update({f"{k}_dram_bytes": int(v[1]) for k, v in bw.items()})
                e["backward_dram_bytes"] = int(sum(v[1] for v in bw.values()))
        traffic[f"C{c}"] = e
        open(os.path.join(PROF, f"{rnd}_launches_c{c}.txt"), "w").write("\n".join(lines) + "\n")
        for k in ("tc_fused", "tc_gemm1", "tc_gemm2", "ir_kernel", "softmax", "tc_gemm2_fi", "tc_bwd_ds", "tc_bwd_dkdv"):
            rep = os.path.join(OUT, f"full_c{c}_{k}.ncu-rep")
            if os.path.exists(rep):
                s = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "ncu_summary.py"), rep, "25"],
                                   capture_output=True, text=True).stdout
                open(os.path.join(PROF, f"{rnd}_full_c{c}_{k}.txt"), "w").write(
                    f"# ncu --set full --clock-control none, tools/run_layer.py {c} (second launch)\n" + s)
    json.dump(traffic, open(os.path.join(PROF, "ncu_traffic.json"), "w"), indent=1)
    print(json.dumps(traffic, indent=1))


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "r1")
