"""B200-native GPU Merkle-tree checkpoint de-duplication (Tan et al., ICPP'23)."""
