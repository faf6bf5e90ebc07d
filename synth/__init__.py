"""Seeded synthetic input generators shared by the CUDA path and the CPU oracle.

This package holds NO arithmetic of the method (no sampling, no unique, no
gather).  It only produces the inputs the paper's workloads are shaped like
(Table II; SURVEY.md section 8(d) "Generator formulas"):

* a row-local power-law CSR graph (``graph``): the adjacency of node v is a
  pure function of (graph_seed, v), so any row can be regenerated on the host
  for the oracle without materialising the whole graph;
* procedural node features (``features``): bits = f(feat_seed, v, c);
* seed nodes per global batch and the per-batch RNG seed (``seeds``);
* the five BASELINE.json configurations as named presets (``presets``).

Both sides (``paper_conf_sc_yanglql22_b200`` and ``oracle``) may import this
package; neither imports the other.
"""

from . import hashing, graph, features, seeds, presets  # noqa: F401
