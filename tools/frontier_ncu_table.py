"""Per-algorithm table of an ncu --set full capture of every k_relax_fq launch
(tools/ncu_summary.py JSON lines, launches in the order frontier_probe.py runs them: BFS, SSSP,
SSWP, CC), with the processed-arc counts of the same graphs (tigr_stats.edges_processed).

    python tools/frontier_ncu_table.py summary.jsonl bfs=6:266302675 sssp=8:413558789 ...
"""
import json
import sys


def unit_scale(v, u):
    return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ms": 1e-3, "us": 1e-6, "ns": 1e-9,
                "msecond": 1e-3, "usecond": 1e-6, "nsecond": 1e-9}.get(u, 1)


def main():
    rows = [json.loads(x) for x in open(sys.argv[1]) if x.startswith("{")]
    print("algo | launches | ms | DRAM GB/s | L1 sectors/request | L1 sectors/processed arc | warp eff. | "
          "heaviest: ms, L2 hit %, occupancy %, regs, top stall")
    i = 0
    for spec in sys.argv[2:]:
        algo, rest = spec.split("=")
        nl, arcs = (int(x) for x in rest.split(":"))
        rs = rows[i:i + nl]
        i += nl
        t = sum(unit_scale(r["duration"], r["duration_unit"]) for r in rs)
        dram = sum(unit_scale(r["dram_read"], r["dram_read_unit"]) + unit_scale(r["dram_write"], r["dram_write_unit"])
                   for r in rs)
        sec = sum(r["l1_ld_sectors"] for r in rs)
        req = sum(r["l1_ld_requests"] for r in rs)
        inst = sum(r["inst"] for r in rs)
        weff = sum(r["threads_per_inst"] * r["inst"] for r in rs) / inst / 32
        h = max(rs, key=lambda r: unit_scale(r["duration"], r["duration_unit"]))
        st = next(iter(h["top_stalls"].items()))
        print(f"{algo} | {nl} | {t * 1e3:.3f} | {dram / t / 1e9:.0f} | {sec / req:.1f} | {sec / arcs:.2f} | "
              f"{100 * weff:.1f}% | {unit_scale(h['duration'], h['duration_unit']) * 1e3:.3f}, "
              f"{h['l2_hit_pct']:.1f}, {h['occupancy_pct']:.1f}, {h['regs']:.0f}, {st[0]} {st[1]}%")


if __name__ == "__main__":
    main()
