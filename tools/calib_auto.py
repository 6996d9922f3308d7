import os, sys, json
sys.path.insert(0, '/root/repo')
import paper_conf_ipps_hainscobr11_b200 as swp
from workloads import gen
from workloads.matrices import BLOSUM62
lens = gen.sp_lengths(540_000, seed=2)
db = gen.build_database(lens, 2, None)
with swp.SmithWaterman(gen.make_query(144), BLOSUM62, 10, 2) as sw:
    sw.load_db(db.residues, db.offsets)
    for m in (189, 222, 375, 567, 1000):
        sw.set_query(gen.make_query(m))
        os.environ["SW_DEBUG_AUTO"] = "1"
        sw.search(-1)
        os.environ.pop("SW_DEBUG_AUTO")
        for T in (36000, 16384, 8192, 6144, 4096, 3072, 2048):
            sw.search(T); sw.search(T)
            print(json.dumps({"m": m, "T": T, "ms": round(sw.kernel_ms()["search_ms"], 3)}), flush=True)
