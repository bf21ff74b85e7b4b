"""CPU oracle for the Adaptive SGD hot path -- TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously correct fp64 implementation of what the paper's
data-parallel hot path computes (Ma, Rusu, Wu, Sim, IPDPSW'22; the text is
/root/reference/PAPER.md, cited as P:a-b = its lines a..b):

* model.py    -- the local minibatch SGD step of the 3-layer MLP (ReLU,
                 softmax, cross-entropy) over CSR-sparse features
                 (§II, §V-A).
* scaling.py  -- Algorithm 1, batch size scaling.
* merge.py    -- Algorithm 2, normalized model merging.
* routing.py  -- dynamic scheduling / mega-batch routing (Fig. 2).
* metrics.py  -- top-k precision (P@1 = top-1 accuracy).
* adaptive.py -- the whole method over N simulated replicas.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / reference
leg may import anything from this package.  It shares no code with the CUDA
path (paper_conf_ipps_marws22_b200/); the only common module is synth/, which
draws the seeded inputs and holds none of the method's arithmetic.

Parity pins (tests/test_oracle_*.py): finite differences and PyTorch CPU fp64
autograd for the step; torch.optim.SGD for the N=1, gamma=0 trajectory;
exact-rational golden vectors and invariants for Alg. 1 / Alg. 2; the Fig. 2
worked example for routing; brute-force sorting for P@k.  Time-to-P@1 is
"parity unpinned" (the paper prints no values).
"""
