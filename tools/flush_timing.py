"""Per-phase clock64 breakdown of k_flush (build exp/lib_ftime.so with -DGG_FLUSH_TIMING)."""
import ctypes, os, subprocess, sys, json
import numpy as np
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
os.environ["GGRID_LIB"] = os.path.join(ROOT, "exp", "lib_ftime.so")
sys.path.insert(0, ROOT)
sys.argv = [sys.argv[0], "--parity", "0", "--queries", "1024", "--repeat", "2"] + sys.argv[1:]
import runpy
runpy.run_path(os.path.join(ROOT, "tools", "c3_flush_roofline.py"), run_name="__main__")
import paper_conf_icde_li0qhdy18_b200 as gg
L = gg.lib()
buf = (ctypes.c_ulonglong * 8)()
L.ggrid_debug_flush_timing(buf)
names = ["loop_top->gather_start (pipeline + prev tail)", "gather", "match stream", "count+clear", "scan", "out+vobj+scatter+tail"]
tot = sum(buf[:6])
for i, n in enumerate(names):
    print(f"{n:45s} {buf[i]/1e6:10.1f} Mcyc  {100*buf[i]/tot:5.1f}%")
