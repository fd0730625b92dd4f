"""CPU oracle for the STRONGHOLD working-window engine -- TEST INFRASTRUCTURE.

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg and
`--impl reference`) may import anything from here.  The product package
paper_conf_sc_sunwqyhxw22_b200 never imports it and shares no code with it.

Parity status per function:
  gpt_oracle.forward_backward  pinned: finite differences + torch.nn.functional/autograd fp64
                               + special cases (seq=1 attention, zero head => ln V, const-row LN)
  gpt_oracle.adamw_update      pinned: constant-gradient closed form + torch.optim.AdamW fp64
  gpt_oracle.global_grad_norm  pinned: brute-force scalar sum on tiny input
  autotune_oracle.solve_window pinned: homogeneous closed forms + brute-force feasibility
"""
