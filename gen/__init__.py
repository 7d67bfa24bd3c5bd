"""Seeded synthetic workloads (pattern sets + input byte streams).

This package holds none of the method's arithmetic: it only draws seeded
random pattern strings and byte streams shaped like the paper's benchmark
suites (Table 1; inputs of P:L431), per the recipes in
DESIGN.md Sec. "Input recipe" / SURVEY.md Sec. 8(d).  Both the oracle side
(tests, bench cpu_baseline) and the CUDA side (tests, bench) consume it.
"""
from .workloads import (CONFIGS, amino_lines, brill_patterns, clamav_brill_patterns, clamav_patterns,  # noqa: F401
                        dotstar_input, dotstar_patterns, dotstar_protomata_patterns, fuzz_pattern, fuzz_text,
                        make_config, multi_input, multi_patterns, protomata_patterns, snort_input, snort_patterns,
                        text_input, tiny_input, tiny_patterns)
