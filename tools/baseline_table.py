#!/usr/bin/env python3
"""Render BASELINE.md section 7's table from a directory of bench.py JSON lines."""
import glob
import json
import os
import sys

NAMES = {1: "1 (1 k x 4 KB-1 MB, 30% dup)", 2: "2 (1 M x 256 B-4 KB, 60% dup)", 3: "3 (10 k x 1 MiB near-dup)",
         4: "4 (1 k x 16-64 MiB, 40.9 GB)", 5: "5 (2 M mixed, 63.4 GB, 10 k sites)"}
MODES = [("", "default"), ("_tp", "two-pass (forced)"), ("_pf", "prefilter"), ("_db0", "digest_bits=0")]


def main(d, prefix):
    out = ["| Config | P | mode (round 0) | payload GB/s | ms/step | alg GB/s | % of 8 TB/s | % of read ceiling (7391) "
           "| dominant kernel: frac of copy peak | e2e GB/s (pinned host) | oracle GB/s (1 core) | parity |",
           "|---|---|---|---|---|---|---|---|---|---|---|---|"]
    for k in range(1, 6):
        for suf, mode in MODES:
            f = os.path.join(d, f"{prefix}_c{k}{suf}.json")
            if not os.path.exists(f):
                continue
            j = json.loads(open(f).read().strip().splitlines()[-1])
            alg = j["path_alg_gbs"]
            r0 = j["config"].get("round0", "")
            e2e = j["e2e"]["value"] if j.get("e2e") else "-"
            cpu = j["cpu_baseline"]["value"] if j.get("cpu_baseline") else "-"
            out.append(f"| {NAMES[k]} | 1 | {mode}: {r0} | {j['value']:.0f} | {j['ms_per_step']:.3f} | {alg:.0f} | "
                       f"{alg / 8000 * 100:.1f}% | {alg / 7391 * 100:.1f}% | {j['roofline']['kernel']} "
                       f"{j['roofline']['frac']:.2f} | {e2e} | {cpu} | bit-exact (full size) |")
    print("\n".join(out))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])
