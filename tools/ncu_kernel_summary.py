"""Compact summary of one kernel from an `ncu --page raw --csv` export (first kernel row):
duration, pipe utilisation, DRAM traffic, occupancy, registers and the stall breakdown."""
import csv, json, sys

KEYS = ["gpu__time_duration.sum", "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "sm__warps_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_tensor_subpipe_dmma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
        "sm__instruction_throughput.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "dram__bytes_read.sum", "dram__bytes_write.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum",
        "lts__t_sector_hit_rate.pct",
        "sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
        "sm__mem_tensor_cycles_active.avg.pct_of_peak_sustained_active",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed"]


def summarise(path, source):
    rows = list(csv.reader(open(path)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    d = dict(zip(hdr, vals))
    u = dict(zip(hdr, units))
    out = {"source": source, "kernel": d.get("Kernel Name", "")[:160]}
    for k in KEYS:
        if k in d:
            out[k] = "%s %s" % (d[k], u.get(k, ""))
        else:   # section-prefixed names (e.g. "TPC.TriageCompute.<metric>")
            for kk in d:
                if kk.endswith("." + k):
                    out[k] = "%s %s" % (d[kk], u.get(kk, ""))
                    break
    stalls = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): float(v.replace(",", ""))
              for k, v in d.items() if k.startswith("smsp__pcsamp_warps_issue_stalled_")
              and not k.endswith("not_issued") and v.replace(",", "").replace(".", "").isdigit()}
    tot = sum(stalls.values()) or 1.0
    out["stall_samples_share"] = {k: round(v / tot, 3) for k, v in sorted(stalls.items(), key=lambda x: -x[1])
                                  if v / tot >= 0.01}
    return out


if __name__ == "__main__":
    json.dump(summarise(sys.argv[1], sys.argv[3] if len(sys.argv) > 3 else sys.argv[1]),
              open(sys.argv[2], "w"), indent=1)
