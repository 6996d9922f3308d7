"""Timing probe for an alternative build of the library (A/B experiments; scores not checked):
python tools/variant_probe.py LIB.so m menu len [n_residues]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_hainscobr11_b200 as swp  # noqa: E402

swp.load_library(sys.argv[1])
sys.argv = [sys.argv[0]] + sys.argv[2:]
exec(open(os.path.join(ROOT, "tools", "uniform_probe.py")).read())
