"""CPU oracle for exact-greedy GBDT (TEST INFRASTRUCTURE ONLY; see oracle/gbdt_oracle.c)."""
