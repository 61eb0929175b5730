import sys, os
sys.path.insert(0, os.getcwd())
import paper_conf_ppopp_mccoyp24_b200 as G
G.gallatin_init(16 << 30)
print(G.gallatin_probe(11, 1 << 24, 148) if hasattr(G, "gallatin_probe") else "no probe fn")
G.gallatin_destroy()
