"""CPU oracle for AvgPipe's elastic-averaging step and advance-forward schedule.

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import or call
anything in this package.  The product path (``paper_conf_ppopp_chen0qz23_b200``,
its C-ABI library and CUDA kernels) never imports it, and this package never
imports the product: the two share no code, headers, helpers or constants.

Paper: Chen, Xu, Qian, Zhou, "Elastic Averaging for Efficient Pipelined DNN
Training" (AvgPipe), PPoPP'23.  Citations ``P:<line> §<sec>`` refer to the
paper text line and section.

Modules
  ea_oracle  float64 numpy implementation of the per-iteration elastic
             averaging step (§3.2), step by step in the paper's order.
  schedule   the advance-forward-propagation micro-batch order
             (Algorithm 1, §4.2) and its AFAB / 1F1B special cases
             (§4.1).

Pinning status: every function here is pinned by
``tests/test_oracle_pins.py`` / ``tests/test_schedule_oracle.py`` to closed
forms, library routines (torch.optim.SGD), exact-rational brute force and the
paper's worked example (Fig. 7, tests/golden/fig7_schedule.json), except the
statement "communication blocks AFAB 2x, 1F1B 9x", which needs the
figure's durations: parity unpinned, and nothing in the oracle depends on it.
"""
