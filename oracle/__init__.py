"""CPU oracle (test infrastructure only). See oracle/orc.h."""
