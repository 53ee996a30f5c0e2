#!/usr/bin/env python3
"""One 16M-node narrow batch of the corpus (the e2e / bench batch shape), built once after one
warm-up build: the target of the heavy-round ncu captures (scripts/gpu_ncu_heavy.sh)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_yuwobby20_b200 as gd
from paper_conf_ipps_yuwobby20_b200 import corpus
from synth import generator as G
n = 1000
sizes = G.corpus_sizes(n)
wide = [G.corpus_config(i).q_cap > 64 for i in range(n)]
plan = corpus.plan_corpus(sizes, wide, 1, node_budget=16_000_000)
batch = [b for b in plan.batches[0] if not any(wide[i] for i in b)][int(sys.argv[1]) if len(sys.argv) > 1 else 0]
apps = [G.corpus_app(i) for i in batch]
h = gd.load(apps, stream=torch.cuda.current_stream().cuda_stream)
for it in range(int(os.environ.get("BUILDS", "2"))):
    st = h.build(byte_model=False)
    print(f"build {it}: {st['fixpoint_ns'] / 1e6:.1f} ms fixpoint, {st['rounds']} rounds, {st['node_visits']} visits,"
          f" {sum(a.n_nodes for a in apps)} nodes, {len(apps)} apps", flush=True)
