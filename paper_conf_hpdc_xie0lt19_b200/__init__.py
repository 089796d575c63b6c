"""B200-native LDA collapsed-Gibbs sweep (CuLDA_CGS hot path)."""
