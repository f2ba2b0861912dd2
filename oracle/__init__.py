"""CPU oracle for derived-field generation (Harrison et al., SC-companion 2012).

TEST INFRASTRUCTURE ONLY.  Nothing in the product path
(``paper_conf_sc_harrisonnmjc12_b200``) may import, call or link anything in
this package.  Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs use it.

What it is: a plain, slow, obviously-correct re-statement of the method in
``/root/reference/PAPER.md`` (cited as ``L<n>``):

* ``oracle.lang``      -- expression language, parse tree, dataflow network
                          specification with constant de-duplication and
                          limited CSE, canonical DAG text (L66-L76, L84-L85).
* ``oracle.evaluate``  -- literal whole-array evaluation of every primitive in
                          the field type T, in network order (L86, L97-L105,
                          Eq. 1-3 at L136-L148); grad3d per DESIGN.md reading R1.
* ``oracle.model``     -- the strategies' device-event counts (Table II,
                          L271-L289) and device-memory high-water model
                          (Fig. 2).
* ``oracle.halo``      -- z-slab decomposition and ghost-plane maps (the
                          ghost data of L255 / L315, reading R12).

It shares no code with the CUDA path; the only common module is ``synth``
(seeded input generators, no method arithmetic).

Pins (tests/test_oracle_*.py, ``-m "not gpu"``): Table II (27 integers),
Fig. 2 (3/4/5 arrays), closed-form fields (linear, rotation, strain, shear,
quadratic) bit-exact on dyadic meshes, numpy.gradient on uniform meshes,
vorticity/Q identities, exact-rational brute force on 4^3 meshes.
Parity unpinned: nothing in this package is unpinned; the synthetic
RT-like field values have no paper values.
"""

from . import lang, evaluate, model, halo  # noqa: F401
