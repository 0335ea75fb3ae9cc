"""Workloads: fused-operator descriptions and seeded synthetic inputs.

This package is the ONLY code shared by the product path
(``paper_conf_cgo_bastoulzrlsjfjc22_b200``) and the oracle (``oracle/``).  It
holds no arithmetic of the method: it writes fused operators down in a plain
dict form and draws seeded random inputs.  Both sides parse the dict form with
their own code.

Description format (a plain dict)::

    {
      "name":    "cfg1_add_mul_relu",
      "loops":   {"a": 4, "b": 8, "c": 16},          # loop name -> extent E_l
      "tensors": {"x": {"shape": [4, 8, 16], "dtype": "f32", "role": "in",
                        "strides": None,             # optional, elements
                        "init": ("uniform", -1, 1, seed)},
                  ...},
      "stmts": [
        {"kind": "assign",                            # or "reduce"
         "op": "sum",                                 # reduce only: sum | max
         "loops": ["a", "b", "c"],                    # outermost first
         "write": ("out", ["a", "b", "c"]),
         "reads": [("x", ["a", "b", "c"]), ("bias", ["c"]), ...],
         "expr":  [("load", 0), ("load", 1), ("add", 0, 1), ...],
         "finalize": [("acc",), ("const", 768.0), ("div", 0, 1)]},  # reduce only
      ],
    }

Roles: in, out, inout, temp (an intermediate of the fused operator).
An index entry is a loop name (iterator, coefficient 1), an int (constant) or
a ``(loop, offset)`` pair — the access functions of PAPER.md P:355 ("either a
constant or an affine form where only one loop iterator is present with
coefficient 1").  ``expr`` is a DAG in topological order; operands are indices
of earlier nodes, ``("load", k)`` reads ``reads[k]``, ``("cast", a, dtype)``
rounds to a dtype; the statement value is the last node.  Statement semantics
are defined in ``include/fop.h``.
"""

from .configs import (CONFIGS, cfg1, cfg1_bias_b, cfg2, cfg3, cfg4a, cfg4b,
                      fig2_running_example, transpose2d, nhwc_to_nchw, cfg2_nhwc, bias_add_rows, algorithmic_bytes,
                      elem_size, N4, N3, ODD)
from .inputs import (make_inputs, alloc_outputs, tensor_span, tensor_strides,
                     contiguous_strides, NP_DTYPE)

__all__ = [
    "CONFIGS", "cfg1", "cfg1_bias_b", "cfg2", "cfg3", "cfg4a", "cfg4b",
    "fig2_running_example", "transpose2d", "nhwc_to_nchw", "cfg2_nhwc", "bias_add_rows", "algorithmic_bytes", "elem_size", "N4", "N3", "ODD",
    "make_inputs", "alloc_outputs", "tensor_span", "tensor_strides",
    "contiguous_strides", "NP_DTYPE",
]
