"""profiles/traffic.json from the ncu --set full raw CSVs of one capture round:
dram__bytes_read.sum + dram__bytes_write.sum of one segment-kernel launch x column tiles
per step, plus the unit utilisations bench.py quotes in roofline.units.
Usage: python tools/make_traffic.py TAG [dir]   (reads DIR/ncu_TAG_<wl>_k<K>_raw.csv)"""
import csv, json, os, sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
# (workload-kK, B dtype) -> column tiles per step (bf16: 128-column tiles of 256 B)
TILES = {("reddit-k64", "f32"): 1, ("reddit-k256", "f32"): 4, ("products-k128", "f32"): 2,
         ("rmat-k64", "f32"): 1, ("products-k128", "bf16"): 1}
UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}


def main(tag, d):
    out = {}
    units = {}
    for (wl, dt), tiles in TILES.items():
        name, k = wl.split("-k")
        path = os.path.join(d, "ncu_%s_%s_k%s%s_raw.csv" % (tag, name, k, "" if dt == "f32" else "_" + dt))
        if not os.path.exists(path):
            continue
        rows = list(csv.reader(open(path)))
        hdr, un, val = rows[0], rows[1], rows[2]
        get = lambda m: float(val[hdr.index(m)])
        b = lambda m: get(m) * UNIT[un[hdr.index(m)]]
        key = "%s-%s-atomic" % (wl, dt)
        out[key] = int(round((b("dram__bytes_read.sum") + b("dram__bytes_write.sum")) * tiles))
        units[key] = {
            "lts_throughput_pct": round(get("lts__throughput.avg.pct_of_peak_sustained_elapsed"), 1),
            "l2_hit_pct": round(get("lts__t_sector_hit_rate.pct"), 1),
            "dram_throughput_pct": round(get("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"), 2),
        }
    out["_note"] = ("ncu --set full, %s: dram__bytes_read.sum + dram__bytes_write.sum of one "
                    "segment-kernel launch x column tiles per step (one cold-cache launch "
                    "per tile)" % tag)
    out["_units"] = units
    with open(os.path.join(ROOT, "profiles", "traffic.json"), "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else os.path.join(ROOT, "gpurun_out"))
