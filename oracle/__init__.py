"""ORACLE -- test infrastructure only.

A plain, slow, obviously-correct CPU implementation of what DeepPlan's cold-start hot
path computes, written from /root/reference/PAPER.md (cited as P:<line>) and the
readings listed in DESIGN.md §3 (= SURVEY §8(c)).

* ``oracle.forward``  -- fp64 numpy transformer forward (BERT / RoBERTa / GPT-2, HF
  semantics).  DeepPlan only changes WHERE weights are read from, so the
  oracle of the forward is the plain definition.
* ``oracle.units``    -- planning units and their byte counts (Table 1
  closed forms).
* ``oracle.planner``  -- pipeline simulator (P1), Algorithm 1, greedy
  "initial approach", PT partition, exhaustive search.
* ``oracle.serving``  -- discrete-event replay of the serving policy.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_eurosys_jeongba23_b200``) never imports it, and this package never
imports the product path.  Inputs come from ``synth`` (data only).
"""
