#!/usr/bin/env python
"""Render `bench.py --workload sweep` JSONL rows as the profiles/ markdown table.
Usage: sweep_md.py rows.jsonl [peak_gbs]"""
import json
import sys

COLS = ["config", "payload B", "kernel", "pack us", "unpack us", "pack GB/s", "unpack GB/s", "frac",
        "pack vs copy", "unpack vs copy", "graph pack/unpack us", "sector frac", "oracle 1t GB/s",
        "oracle all-core GB/s"]


def main():
    rows = [json.loads(x) for x in open(sys.argv[1]) if x.startswith("{") and '"config"' in x]
    rows = [r for r in rows if "pack_us" in r]
    print("| " + " | ".join(COLS) + " |")
    print("|" + "|".join(["---"] + ["---:"] * (len(COLS) - 1)) + "|")
    for r in rows:
        g = r.get("graph_pack_us")
        graph = f"{g} / {r.get('graph_unpack_us')}" if g is not None else ""
        cells = [r["config"], r["payload"], r["kernel"], r["pack_us"], r["unpack_us"], r["pack_gbs"],
                 r["unpack_gbs"], r["pack_frac_hbm"], r["pack_vs_copy"], r["unpack_vs_copy"], graph,
                 r.get("pack_sector_aware_frac", ""), r.get("oracle_1t_gbs", ""), r.get("oracle_mt_gbs", "")]
        print("| " + " | ".join(str(c) for c in cells) + " |")
    if rows and "oracle_cores" in rows[0]:
        print(f"\noracle host cores: {rows[0]['oracle_cores']}")


if __name__ == "__main__":
    main()
