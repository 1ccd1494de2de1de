#!/usr/bin/env python
"""Joins the ncu range-replay CSV of tools/counters.py with its case list into a markdown table of
counters per payload byte (PCIe read/write, DRAM read/write) and the range's rates.

    python tools/counters_table.py gpurun_out/counters.csv gpurun_out/counter_cases.json > profiles/rNN_counters_crossover.md
    python tools/counters_table.py gpurun_out/counters_tma.csv probe_tma     # tools/probe_tma ranges (1 GiB each)
"""
import csv
import json
import sys


def load(csv_path, cases_path):
    rows = [r for r in csv.reader(open(csv_path)) if r and r[0] != "" and not r[0].startswith("==")]
    head = rows[0]
    by = {}
    for r in rows[1:]:
        d = dict(zip(head, r))
        v = float(d["Metric Value"].replace(",", ""))
        unit = d["Metric Unit"]
        if unit in ("nsecond", "ns"):
            v *= 1e-9
        elif unit in ("usecond", "us"):
            v *= 1e-6
        elif unit in ("msecond", "ms"):
            v *= 1e-3
        elif unit == "Kbyte":
            v *= 1e3
        elif unit == "Mbyte":
            v *= 1e6
        elif unit == "Gbyte":
            v *= 1e9
        by.setdefault(int(d["ID"]), {})[d["Metric Name"]] = v
    if cases_path == "probe_tma":
        names = ["ce_h2d", "ce_d2h", "ldg_h2d", "stg_d2h", "tma_h2d", "tma_d2h"]
        cases = [{"mechanism": nm, "chunk": 0, "phase": "h2d" if "h2d" in nm else "d2h", "payload": 1 << 30}
                 for nm in names]
    else:
        cases = json.load(open(cases_path))
    assert len(cases) == len(by), (len(cases), len(by))
    return [dict(c, **by[i]) for i, c in enumerate(cases)]


def main():
    recs = load(sys.argv[1], sys.argv[2])
    print("| chunk | phase | mechanism | range ms | payload GB/s | PCIe rd B/B | PCIe wr B/B | PCIe GB/s (rd+wr) | DRAM rd B/B | DRAM wr B/B |")
    print("|---|---|---|---|---|---|---|---|---|---|")
    for r in sorted(recs, key=lambda r: (r["chunk"], r["phase"], r["mechanism"])):
        P = r["payload"]
        t = r["gpu__time_duration.sum"]
        pr, pw = r["pcie__read_bytes.sum"], r["pcie__write_bytes.sum"]
        print(f"| {r['chunk'] >> 10} KiB | {r['phase']} | {r['mechanism']} | {t * 1e3:.2f} | {P / t / 1e9:.2f} | "
              f"{pr / P:.4f} | {pw / P:.4f} | {(pr + pw) / t / 1e9:.2f} | {r['dram__bytes_read.sum'] / P:.4f} | "
              f"{r['dram__bytes_write.sum'] / P:.4f} |")


if __name__ == "__main__":
    main()
