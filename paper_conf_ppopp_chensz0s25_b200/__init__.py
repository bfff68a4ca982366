"""B200-native V:N:M sparse-tensor-core SpMM for reordered graphs (PPoPP'25 hot path)."""
