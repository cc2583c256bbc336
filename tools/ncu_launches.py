"""Summarise an ncu launch-list CSV (--metrics gpu__time_duration.sum[,dram bytes]) by kernel family."""
import collections, csv, json, sys

SCALE_T = {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3}
SCALE_B = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "B": 1, "KB": 1e3, "MB": 1e6, "GB": 1e9}


def summarise(path, source):
    rows = [r for r in csv.reader(open(path)) if len(r) > 10]
    hdr = rows[0]
    ki, mi, vi, ui, idi = (hdr.index(k) for k in ("Kernel Name", "Metric Name", "Metric Value", "Metric Unit", "ID"))
    per = collections.defaultdict(dict)
    for r in rows[1:]:
        v = float(r[vi].replace(",", ""))
        if r[mi] == "gpu__time_duration.sum":
            per[r[idi]]["us"] = v * SCALE_T[r[ui]]
        elif r[mi].startswith("dram__bytes"):
            per[r[idi]]["bytes"] = per[r[idi]].get("bytes", 0.0) + v * SCALE_B[r[ui]]
        per[r[idi]]["name"] = r[ki].split("(")[0].replace("void ", "").split("<")[0]
    fam = collections.defaultdict(lambda: [0, 0.0, 0.0])
    for d in per.values():
        f = fam[d["name"]]
        f[0] += 1
        f[1] += d.get("us", 0.0)
        f[2] += d.get("bytes", 0.0)
    tot = sum(v[1] for v in fam.values())
    return {"source": source, "launches": len(per),
            "families": {k: {"launches": v[0], "time_us": round(v[1], 1), "share": round(v[1] / tot, 4),
                             "dram_GB": round(v[2] / 1e9, 3),
                             "GBps": round(v[2] / (v[1] * 1e-6) / 1e9, 1) if v[1] and v[2] else None}
                         for k, v in sorted(fam.items(), key=lambda x: -x[1][1])}}


if __name__ == "__main__":
    out = summarise(sys.argv[1], sys.argv[3] if len(sys.argv) > 3 else sys.argv[1])
    json.dump(out, open(sys.argv[2], "w"), indent=1)
    print(json.dumps(out["families"], indent=1))
