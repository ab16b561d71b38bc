"""ORACLE package — test infrastructure only (see oracle/sq_oracle.c)."""
