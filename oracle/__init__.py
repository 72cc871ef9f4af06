"""ORACLE — test infrastructure only. NOT part of the product path.

Plain, slow, obviously correct CPU implementation of what the hot path
computes, written from PAPER.md (Kasagi, Nakano, Ito, ICPP 2013). Only
``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import, call, link or execute anything here.
The product (``paper_conf_icpp_kasagini13_b200`` + ``libperm.so``) never
imports this package, and this package never imports the product: they
share only the seeded input generators in ``workloads/``.

Modules (each function cites the passage it follows):

* ``apply``        the definition b[P(i)] = a[i] (L361), D-/S-designated (L365, L373)
* ``hmm``          DMM bank / UMM address-group round classification (L201-L215)
* ``distribution`` D_w(P) (L389-L401, Lemma 4)
* ``konig``        König edge colouring by alternating paths (Thm 6)
* ``planner``      reference scheduled-permutation planner (L515-L539, L603-L605)
* ``check``        plan invariants (i)-(vii) (L519, L531-L539); tiled (TLC) and cluster plans
* ``tiled``        the oracle's own TLC / cluster plan builders and executors (L531-L539 over
                   tiles; Lemma 8's transposes as chunk scatters / block exchanges)
* ``emulate``      paper-faithful R,T,R,T,R with a Table I round counter (L409-L533, L681)
* ``c/apply_ref.c`` the definition as a plain C loop, for CPU timing only

Pins (tests/test_oracle_*.py) tie each function to something other than
itself: Fig. 3/4/6 fixtures, closed forms of D_w, Table III's D_w band,
Table I round counts, brute force over all permutations at tiny n.
"""
