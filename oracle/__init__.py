"""CPU ORACLE — test infrastructure only.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference leg may import or execute anything under oracle/.  The product path
(paper_conf_sc_tangtrwckgtw13_b200/, libbro.so) never calls it, and this
package never imports the product; the two share no code.  Inputs come from
the neutral generator package gen/.

What it computes (citations are PAPER.md line numbers, "P:Lnnn"):

  spmv.py     plain SpMV  y_i = sum_j a_ij x_j  over stored entries, in higher
              precision (longdouble for fp64 data, fp64 for fp32 data), plus
              S_i = sum_j |a_ij||x_j| for the parity tolerance (the
              definition of y = A.x).
  hyb.py      ELLPACK arrays, HYB split with the "less than a third"
              rule (pinned by the worked split at P:L79), ELLPACK-R
              row_length.
  bro_ell.py  BRO-ELL encoder, step by step as P:L103-116 (delta, slices,
              num_col, per-column bit_alloc, padding bits b_p, multiplexing),
              and the decoder as a literal transcription of Algorithm 1
              (P:L128-138).
  bro_coo.py  BRO-COO encoder/decoder.  Its 2D interval
              arrangement follows DESIGN.md reading R13 because Fig. 2 is not
              in the text: the LAYOUT IS PARITY UNPINNED against the paper
              (pinned only by round trips and by SpMV through the decoder).
  metrics.py  space savings eta = 1 - C/O and compression ratio
              kappa = 1/(1-eta).
  bar.py      BRO-aware reordering: Eqn (1)-(3) and Algorithm 2.
  value_index.py  value indexing of the BRO-ELL values: the "value data
              compression" the conclusion names as future work, by
              the value-index method of the work it cites ([16]):
              distinct bit patterns + 1- or 2-byte codes in the slot layout
              (reading R28; pinned by matrix A by hand, the stencil
              closed form and a bitwise round trip).

Every pin (tests/test_oracle_*.py, tests/golden/) ties these functions to
something other than themselves: the paper's worked example, closed forms,
brute force on tiny inputs, scipy.sparse, round trips.
"""
