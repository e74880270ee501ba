import time, torch, sys
sys.path.insert(0, '.')
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G, synth
dev = torch.device('cuda:0')
w = synth.WORKLOADS['reddit']
s, d = w.edges(0, dev)
torch.cuda.synchronize()
for i in range(3):
    t = time.perf_counter()
    g = G.granii_graph_csr_create(w.n, s, d, G.ADD_SELF_LOOPS | G.SYMMETRIZE)
    print(i, 'total ms %.1f' % ((time.perf_counter() - t) * 1e3), G.granii_graph_timings(g))
    del g
