"""Chunk-size sweep of sw_search_stream on C2: the host-resident database is
cut into chunks that are sorted/packed/uploaded while the previous chunk is searched.  Prints
one JSON line per chunk size (wall seconds of the blocking call, GCUPS) and the resident
search_batch time for comparison.
    python tools/stream_chunk_sweep.py [--config C2]"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_ipps_hainscobr11_b200 as swp  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--chunks", type=int, nargs="*", default=[24, 25, 26, 27, 28], help="log2 chunk sizes")
    a = ap.parse_args()
    qs, db, lens_all, mat, rho, sigma, T = bench.make_workload(a.config, 0, 1)
    cells = bench.cells_of(qs, db.total_residues)
    sw = swp.SmithWaterman(qs[0], bench.MATRICES[mat], rho, sigma)
    sw.load_db(db.residues, db.offsets)
    sw.search_batch(qs, T)
    t0 = time.perf_counter()
    sw.search_batch(qs, T)
    res_s = time.perf_counter() - t0
    print(json.dumps({"mode": "resident", "seconds": round(res_s, 4), "gcups": round(cells / res_s / 1e9, 1)}), flush=True)
    if os.environ.get("SW_AUTOTUNE") == "0":
        print(json.dumps({"note": "SW_AUTOTUNE=0: planner's model choice only"}), flush=True)
    for lg in a.chunks:
        chunk = 1 << lg
        sw.search_stream(db.residues, db.offsets, T, chunk, queries=qs)
        ts = []
        for _ in range(a.reps):
            t0 = time.perf_counter()
            sw.search_stream(db.residues, db.offsets, T, chunk, queries=qs)
            ts.append(time.perf_counter() - t0)
        s = min(ts)
        print(json.dumps({"mode": "stream", "chunk_residues": chunk, "seconds": round(s, 4),
                          "gcups": round(cells / s / 1e9, 1)}), flush=True)


if __name__ == "__main__":
    main()
