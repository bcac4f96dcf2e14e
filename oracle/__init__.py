"""ORACLE -- TEST INFRASTRUCTURE ONLY.

A plain, slow, obviously-correct CPU implementation of what the paper's
recursive-block SpTRSV computes (Lu, Niu & Liu, ICPP'20, /root/reference/PAPER.md):

  * ``oracle.numeric``   -- Algorithm 1 forward substitution (and its mirror,
    backward substitution for Ux=b), fp64, in plain C (csrc/oracle.c) plus a
    pure-Python twin for tiny inputs.
  * ``oracle.structure`` -- level sets (Alg 2), level-set reordering of every
    triangular (sub)matrix (Sec. 3.3), the recursive / column / row block
    partitions (Alg 4-6), per-block features and the Alg 7 decision tree.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` leg (and ``bench.py --impl reference``) may import anything
from here.  The CUDA library never imports, links or executes it, and this
package imports nothing from the library: the two share no code, headers,
tables or helpers.  The only shared module is ``workloads`` (seeded inputs,
no method arithmetic).

Parity status of every function is recorded in its docstring and in
DESIGN.md section 3; functions without an independent pin say
"parity unpinned".
"""
