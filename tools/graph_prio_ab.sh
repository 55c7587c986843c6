# graph node priorities (default) vs NB_GRAPH_PRIO=0 on the Poisson CG
# (1 and 4 virtual partitions, halo stream) and the FEM CG
python tools/cg_ab.py 512 100 NB_GRAPH_PRIO=0 | tail -1
AB_PARTS=4 python tools/cg_ab.py 512 100 NB_GRAPH_PRIO=0 | tail -1
AB_PARTS=4 AB_HALO=1 python tools/cg_ab.py 512 100 NB_GRAPH_PRIO=0 | tail -1
for i in 1 2; do python tools/fem_time.py 384 20; NB_GRAPH_PRIO=0 python tools/fem_time.py 384 20; done
