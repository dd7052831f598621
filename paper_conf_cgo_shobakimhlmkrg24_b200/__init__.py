"""B200-native ACO instruction scheduler (Shobaki et al., CGO 2024)."""
