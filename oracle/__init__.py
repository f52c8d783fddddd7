"""CPU oracle for the Mobius (Feng et al., ASPLOS '23) fine-tuning step.

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import
anything under ``oracle/``.  The product path (``include/mobius.h``,
``paper_conf_asplos_fengxtwls23_b200/``) shares no code with it.

Plain, slow, obviously-correct implementations written from
``/root/reference/PAPER.md`` (cited as ``P:L<line>``) and the readings of
SURVEY.md §8(c) (cited as ``#<n>`` / ``O-<n>``):

* ``model``    - GPT forward/backward in numpy fp32/fp64 (O-2)
* ``schedule`` - Mobius per-GPU op lists and discrete-event executor (O-3,
                 Fig 4), byte accounting (O-10)
* ``planner``  - Eq 3-11 cost recurrence (O-6), partition brute force (O-7)
* ``milp``     - literal Eq 3-11 MILP via scipy/HiGHS (O-8)
* ``mapping``  - cross mapping Eq 12/13 with exact Fractions (O-9)
* ``adamw``    - host optimizer (O-4, reading #16)

Pins (tests/test_oracle_*.py): finite differences, torch fp64 autograd,
closed forms, Fig 4 / Fig 4b worked examples, brute force vs MILP.
Parity unpinned: prefetch-priority timing (#21) - timing only.
"""
