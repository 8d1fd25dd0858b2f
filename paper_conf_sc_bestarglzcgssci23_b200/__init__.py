"""B200-native A-GNN layer hot path (Besta et al., SC\x2723)."""
