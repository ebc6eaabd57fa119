import os, sys
sys.path.insert(0, '/root/repo'); 
import inputs, paper_conf_sc_doneyhl25_b200 as eim
off, nbr = inputs.config_graph('C2')
ctx = eim.eim_create(0); g = eim.eim_load_graph_csr(ctx, off, nbr)
eim.eim_sample_rrr(ctx, g, 'IC', 1, 0, 2000)
eim.eim_sample_rrr(ctx, g, 'IC', 1, 0, 1 << 18)
print(eim.eim_get_stats(ctx))
